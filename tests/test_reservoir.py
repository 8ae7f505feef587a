"""Reservoir inserts (Section 4.2, P:L189 / P:L248).

CPU: the product's host decision (kde_reservoir_select in libkde) is bit-identical to the
oracle's Algorithm R on the same counter-based draws.
GPU: kde_insert_rows transfers and writes exactly the rows the oracle's reservoir keeps
(last arrival wins within a chunk), resets their karma, and the estimates on the resulting
sample match the oracle."""
import numpy as np
import pytest

import oracle
import paper_conf_sigmod_heimelkm15_b200 as K
import synth


@pytest.mark.parametrize("seed,n_sample,n_seen,k", [(1, 5, 0, 40), (77, 1000, 1000, 4096), (2**63 + 11, 2**22, 3 * 2**22, 2**16),
                                                    (5, 300, 120, 1000), (9, 1 << 28, 1 << 30, 5000)])
def test_product_reservoir_decisions_equal_oracle(seed, n_sample, n_seen, k):
    got = K.kde_reservoir_select(seed, n_sample, n_seen, k)
    ref = oracle.reservoir_slots(seed, n_sample, n_seen, k)
    assert np.array_equal(got, ref)
    if n_seen >= n_sample:
        acc = np.mean(got >= 0)
        expect = np.mean(n_sample / (n_seen + 1 + np.arange(k)))
        assert abs(acc - expect) < 5 * np.sqrt(expect / k) + 1e-3


def test_reservoir_select_rejects_bad_arguments():
    with pytest.raises(K.KDEError):
        K.kde_reservoir_select(1, 0, 0, 3)
    with pytest.raises(K.KDEError):
        K.kde_reservoir_select(1, 10, -1, 3)


@pytest.mark.gpu
def test_insert_rows_follow_the_oracle_reservoir():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    n, d, seed = 3000, 4, 4242
    S0 = synth.make_data("gauss", n, d, seed=60)
    arrivals = synth.make_data("gauss", 40000, d, seed=61)        # arrival ids n+1 .. n+40000
    m = K.KDEModel.create(S0)
    h = m.bandwidth
    m.karma = np.full(n, 3.0)
    n_seen = n
    content = np.arange(1, n + 1)                                   # the sample = arrivals 1..n
    for k in (1, 700, 7000, 32299):
        chunk = arrivals[n_seen - n:n_seen - n + k]
        n_seen2, nw = m.insert_rows(chunk, seed, n_seen, k_init=-1.0)
        assert n_seen2 == n_seen + k
        sl = oracle.reservoir_slots(seed, n, n_seen, k)
        assert nw == len(np.unique(sl[sl >= 0]))
        n_seen = n_seen2
    content = oracle.reservoir_run(seed, n, n_seen)
    all_rows = np.concatenate([S0, arrivals])
    expect = all_rows[content - 1]
    got = m.sample
    assert np.array_equal(got, expect)
    kk = m.karma
    replaced = content > n
    assert np.all(kk[replaced] == -1.0) and np.all(kk[~replaced] == 3.0)
    lo, hi = synth.mixed_workload(expect, 24, seed=62)
    est_o = oracle.estimate(expect, h, lo, hi)
    est = m.estimate(lo, hi)
    assert np.all(np.abs(est - est_o) <= 1e-7 + 1e-5 * np.abs(est_o))


@pytest.mark.gpu
def test_insert_rows_async_matches_sync_and_orders_with_stream_work():
    """kde_insert_rows_async: the same slots and rows as the synchronous call (the host decision is
    identical), the device work in stream order -- a _dev estimate enqueued right after it on the
    same stream sees the inserted rows -- and the caller may overwrite its rows buffer at once."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    n, d, seed = 5000, 3, 99
    S0 = synth.make_data("gauss", n, d, seed=70)
    arrivals = synth.make_data("rect", 60000, d, seed=71)
    ma, ms = K.KDEModel.create(S0), K.KDEModel.create(S0)
    h = ma.bandwidth
    s = torch.cuda.Stream()
    lo, hi = synth.mixed_workload(S0, 8, seed=72)
    dlo, dhi = torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda()
    est = torch.zeros(8, dtype=torch.float64, device="cuda")
    na = nsy = n
    outs = []
    for k in (1000, 20000, 39000):
        buf = arrivals[na - n:na - n + k].copy()
        na2, nwa = K.kde_insert_rows_async(ma.handle, buf, seed, na, k_init=-2.0, stream=s)
        buf[:] = np.nan                                   # the call copied the rows before returning
        with torch.cuda.stream(s):
            K.kde_estimate_batch_dev(ma.handle, dlo, dhi, est, None, stream=s)
            outs.append(est.clone())                      # on s: after the estimate
        nsy2, nws = ms.insert_rows(arrivals[nsy - n:nsy - n + k], seed, nsy, k_init=-2.0)
        assert (na2, nwa) == (nsy2, nws)
        na, nsy = na2, nsy2
        s.synchronize()
        cur = ms.sample
        est_o = oracle.estimate(cur, h, lo, hi)
        assert np.all(np.abs(outs[-1].cpu().numpy() - est_o) <= 1e-7 + 1e-5 * np.abs(est_o))
    torch.cuda.synchronize()
    assert np.array_equal(ma.sample, ms.sample)
    assert np.array_equal(ma.karma, ms.karma)
    ma.close()
    ms.close()


@pytest.mark.gpu
def test_default_torch_stream_orders_dev_calls():
    """torch's default stream (handle 0) reaches the library as cudaStreamLegacy, not as NULL (= the
    model's own stream): a _dev estimate on it is ordered with torch work and CUDA events on it."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    S = synth.make_data("gauss", 1 << 18, 4, seed=80)
    lo, hi = synth.mixed_workload(S, 300, seed=81)
    m = K.KDEModel.create(S)
    ref = m.estimate(lo, hi)
    dlo, dhi = torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda()
    est = torch.full((300,), -1.0, dtype=torch.float64, device="cuda")
    s0 = torch.cuda.current_stream()
    assert s0.cuda_stream == 0
    K.kde_estimate_batch_dev(m.handle, dlo, dhi, est, None, stream=s0)
    got = est.clone()  # torch work on the default stream, after the estimate in stream order
    torch.cuda.synchronize()
    assert np.array_equal(got.cpu().numpy(), ref)
    m.close()
