"""GPU parity of the culled batched scan over the spatially ordered copy of the sample
(scan_cells.cuh, R17) against the fp64 oracle, through the C ABI.

The ordered copy only changes the order in which the (unordered, eq. 2 / P:L98) sum over the
sample is taken and which far (point, box) pairs are skipped as whole cells; the tolerances are
the north star's (see test_gpu_parity.py) plus the R15 culling floor.  Also checked: the index is
rebuilt after every call that changes sample rows, and the result is bitwise repeatable."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

K = pytest.importorskip("paper_conf_sigmod_heimelkm15_b200")

from test_gpu_parity import grad_ok, sel_ok  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    oracle.set_threads(0)


def _boxes(S, q, seed):
    lo2, hi2 = synth.special_boxes(S, seed=seed)
    lo1, hi1 = synth.mixed_workload(S, q - len(lo2), seed=seed + 1)
    return np.concatenate([lo1, lo2]), np.concatenate([hi1, hi2])


def _ref(S, h, lo, hi, kernel):
    if kernel == "epan":
        return oracle.epan_estimate_grad(S, h, lo, hi) + (oracle.epan_grad_abs_scale(S, h, lo, hi),)
    return oracle.estimate_grad(S, h, lo, hi) + (oracle.grad_abs_scale(S, h, lo, hi),)


@pytest.mark.parametrize("kernel,d,n,q", [
    ("gauss", 1, 5003, 256), ("gauss", 2, 40001, 512), ("gauss", 3, 65536, 1300), ("gauss", 5, 30011, 512),
    ("gauss", 8, 20483, 700), ("gauss", 10, 9001, 256), ("gauss", 16, 3001, 300), ("gauss", 4, 200, 256),
    ("epan", 3, 30011, 512), ("epan", 7, 9001, 513)])
def test_cells_match_oracle_and_unordered_scan(kernel, d, n, q):
    """Several box groups (q > 512 for d <= 6, > 256 above), ragged last cell, one-cell samples,
    special boxes (unbounded, empty, far, narrow -> general Phi path), both product kernels."""
    S = synth.make_data("gauss", n, d, seed=80 + d)
    lo, hi = _boxes(S, q, seed=81 + d)
    m = K.KDEModel.create(S)
    if kernel == "epan":
        m.set_kernel("epan")
        m.bandwidth = m.bandwidth * np.sqrt(5.0)
    h = m.bandwidth
    est_o, g_o, mabs = _ref(S, h, lo, hi, kernel)
    assert m.cull and m.cells
    e1, g1 = m.estimate(lo, hi, grad=True)
    sel_ok(e1, est_o)
    grad_ok(g1, g_o, mabs, h)
    sel_ok(m.estimate(lo, hi), est_o)                 # estimate-only kernel
    e1b, g1b = m.estimate(lo, hi, grad=True)          # ownership-ordered sums: bitwise repeat
    assert np.array_equal(e1, e1b) and np.array_equal(g1, g1b)
    assert K.kde_get_cells(m.handle)[1] == 1          # built once, reused while the sample is unchanged
    m.cells = False                                   # the unordered culled scan agrees as well
    e0, g0 = m.estimate(lo, hi, grad=True)
    sel_ok(e0, est_o)
    grad_ok(g0, g_o, mabs, h)
    m.close()


def test_cells_rebuilt_after_sample_changes():
    """replace (host and device paths) bump the sample generation: the next culled batched call
    rebuilds the ordered copy and sees the new rows."""
    import torch
    d, n = 4, 50001
    S = synth.make_data("gauss", n, d, seed=90)
    lo, hi = _boxes(S, 512, seed=91)
    m = K.KDEModel.create(S)
    h = m.bandwidth
    m.estimate(lo, hi)
    assert K.kde_get_cells(m.handle)[1] == 1
    g = synth.rng(92)
    idx = np.sort(g.choice(n, size=3000, replace=False)).astype(np.int64)
    rows = synth.make_data("rect", 3000, d, seed=93)  # rows from another distribution: visible change
    m.replace_points(idx, rows)
    S2 = S.copy()
    S2[idx] = rows
    est_o, g_o, mabs = _ref(S2, h, lo, hi, "gauss")
    e, gr = m.estimate(lo, hi, grad=True)
    assert K.kde_get_cells(m.handle)[1] == 2
    sel_ok(e, est_o)
    grad_ok(gr, g_o, mabs, h)
    # device-pointer replacement
    idx2 = np.sort(g.choice(n, size=1000, replace=False)).astype(np.int64)
    rows2 = synth.make_data("skew", 1000, d, seed=94)
    d_idx = torch.from_numpy(idx2).cuda()
    d_rows = torch.from_numpy(np.ascontiguousarray(rows2)).cuda()
    d_k = torch.tensor([len(idx2)], dtype=torch.int64, device="cuda")
    K.kde_replace_points_dev(m.handle, d_idx, d_rows, d_k, 1.0, stream=torch.cuda.current_stream())
    torch.cuda.synchronize()
    S2[idx2] = rows2
    est_o, g_o, mabs = _ref(S2, h, lo, hi, "gauss")
    e, gr = m.estimate(lo, hi, grad=True)
    assert K.kde_get_cells(m.handle)[1] == 3
    sel_ok(e, est_o)
    grad_ok(gr, g_o, mabs, h)
    # a bandwidth change does not rebuild (the index holds raw coordinates)
    m.bandwidth = h * 1.3
    est_o, _, _ = _ref(S2, h * 1.3, lo, hi, "gauss")
    sel_ok(m.estimate(lo, hi), est_o)
    assert K.kde_get_cells(m.handle)[1] == 3
    m.close()


def test_cells_degenerate_columns_and_duplicates():
    """A constant column (zero range: Morton scale 0), many duplicate points, duplicate boxes."""
    g = synth.rng(95)
    n, d = 20000, 3
    S = np.empty((n, d), np.float32)
    S[:, 0] = 2.5
    S[:, 1] = g.integers(0, 7, n).astype(np.float32)
    S[:, 2] = g.normal(size=n).astype(np.float32)
    h = np.array([0.3, 0.4, 0.2])
    lo, hi = synth.random_boxes(S + g.normal(scale=0.5, size=S.shape).astype(np.float32), 300, seed=96)
    lo = np.concatenate([lo, lo[:212]])
    hi = np.concatenate([hi, hi[:212]])
    m = K.KDEModel.create(S, h)
    est_o, g_o, mabs = _ref(S, h, lo, hi, "gauss")
    e, gr = m.estimate(lo, hi, grad=True)
    sel_ok(e, est_o)
    grad_ok(gr, g_o, mabs, h)
    assert np.array_equal(e[:212], e[300:]) and np.array_equal(gr[:212], gr[300:])
    m.close()


@pytest.mark.parametrize("kind", range(5))
def test_cells_loss_and_grad_all_losses(kind):
    """eq. (5), (14), (18) through the cells scan (768 boxes: full culled CTAs), log bandwidths."""
    S = synth.make_data("gauss", 60000, 5, seed=97)
    lo, hi = synth.mixed_workload(S, 768, seed=98)
    R = synth.make_data("gauss", 120000, 5, seed=97)
    p = synth.true_selectivity_cpu(R, lo, hi)
    lam = 1e-3
    m = K.KDEModel.create(S)
    h = m.bandwidth
    L_o, g_o, est_o = oracle.loss_and_grad(S, h, lo, hi, p, kind, lam, True)
    L_g, g_g, est_g = m.loss_and_grad(lo, hi, p, kind, lam, True, return_est=True)
    sel_ok(est_g, est_o)
    dL = np.array([abs(oracle.loss(kind, lam, e, pp)[1]) for e, pp in zip(est_o, p)])
    mabs = oracle.grad_abs_scale(S, h, lo, hi)
    grad_ok(g_g, g_o, (dL[:, None] * mabs).mean(axis=0) * h, h, np.mean(dL) * h)
    Ltol = np.mean(dL * (1e-7 + 1e-5 * np.abs(est_o))) * 2 + 1e-12
    assert abs(L_g - L_o) <= Ltol + 1e-9 * abs(L_o)
    m.close()


@pytest.mark.parametrize("kernel,d,n", [("gauss", 2, 30011), ("gauss", 5, 70001), ("gauss", 10, 9001),
                                        ("gauss", 16, 3001), ("epan", 4, 30011)])
def test_cells_single_box_matches_oracle(kernel, d, n):
    """q == 1 over the ordered copy (built by a batched call): far cells are not read; every special
    box (unbounded, empty, far, narrow) and a few mixed ones, with and without the gradient.  With
    retained contributions or a stale index the scan falls back to the TMA scan of the sample."""
    S = synth.make_data("gauss", n, d, seed=100 + d)
    lo, hi = _boxes(S, 300, seed=101 + d)
    m = K.KDEModel.create(S)
    if kernel == "epan":
        m.set_kernel("epan")
        m.bandwidth = m.bandwidth * np.sqrt(5.0)
    h = m.bandwidth
    est_o, g_o, mabs = _ref(S, h, lo, hi, kernel)
    m.estimate(lo, hi)                                  # builds the index
    assert K.kde_get_cells(m.handle)[1] == 1
    ks = list(range(len(lo) - 12, len(lo))) + [0, 1, 2, 3, 50, 100]
    for k in ks:
        e1, g1 = m.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
        sel_ok(e1, est_o[k:k + 1])
        grad_ok(g1, g_o[k:k + 1], mabs[k:k + 1], h)
        sel_ok(m.estimate(lo[k:k + 1], hi[k:k + 1]), est_o[k:k + 1])
    e1 = m.estimate(lo[5:6], hi[5:6])
    assert np.array_equal(e1, m.estimate(lo[5:6], hi[5:6]))  # deterministic
    m.set_retain(True)                                  # retained p^(i): the sample-order scan
    e2 = m.estimate(lo[5:6], hi[5:6])
    sel_ok(e2, est_o[5:6])
    c = m.contributions()
    assert np.isclose(c.sum() / n, e2[0], rtol=1e-5, atol=1e-9)
    m.close()


def test_cells_single_box_stale_index_falls_back():
    d, n = 3, 40000
    S = synth.make_data("gauss", n, d, seed=110)
    lo, hi = _boxes(S, 256, seed=111)
    m = K.KDEModel.create(S)
    h = m.bandwidth
    m.estimate(lo, hi)
    idx = np.arange(0, n, 7, dtype=np.int64)
    rows = synth.make_data("rect", len(idx), d, seed=112)
    m.replace_points(idx, rows)                         # index now stale: q == 1 must see the new rows
    S2 = S.copy()
    S2[idx] = rows
    est_o, g_o, mabs = _ref(S2, h, lo, hi, "gauss")
    for k in (0, 9, 77, len(lo) - 1):
        e1, g1 = m.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
        sel_ok(e1, est_o[k:k + 1])
        grad_ok(g1, g_o[k:k + 1], mabs[k:k + 1], h)
    assert K.kde_get_cells(m.handle)[1] == 1            # single-box calls do not rebuild
    m.close()


def test_cells_rebuild_is_deterministic():
    """A rebuild of an unchanged sample (one row rewritten with itself) reproduces the ordered copy
    exactly: the stable radix sort and the fixed reduction order give bitwise-equal estimates."""
    S = synth.make_data("gauss", 70001, 5, seed=120)
    lo, hi = _boxes(S, 600, seed=121)
    m = K.KDEModel.create(S)
    e1, g1 = m.estimate(lo, hi, grad=True)
    m.replace_points(np.array([123], np.int64), S[123:124].copy())
    e2, g2 = m.estimate(lo, hi, grad=True)
    assert K.kde_get_cells(m.handle)[1] == 2
    assert np.array_equal(e1, e2) and np.array_equal(g1, g2)
    m.close()
