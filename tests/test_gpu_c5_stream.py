"""configs[4] at full size: the device-resident streaming step (kde_stream_step_dev:
estimate + gradient + retained p^(i), karma pass + ordered compaction, Listing 1 step,
replacement of flagged points) on d = 10, N = 2^22 -- 1024 karma blocks -- against the
fp64 oracle (SURVEY.md §8(c) "Streaming (C5) is checked in lockstep").

* Lockstep, 200 queries: before every step the oracle is given the GPU's pre-step state
  (sample, h, karma, Listing 1 state) and must reproduce the step's outputs: p_hat
  (1e-7 + 1e-5 rel), dp_hat/dh (1e-4 rel + 1e-4 m_j + the R15 culling floor), karma
  (1e-4 of the step's change), the flag set (identical outside the guard band of
  |K - tau| < 1e-6/(N-1), |p^(i) - thr_20| < 1e-6 thr_20) and h (1e-4 rel).
* Free-running, first 50 queries: the oracle runs the whole loop on its own state from
  the same start; h within 1e-4 rel and identical flag sets at every step.

Where fp64 decides a sign from an estimate (the L1 derivative sign(p_hat - p) when p_hat
is within the selectivity tolerance of p), both sides take the GPU's decision.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

K = pytest.importorskip("paper_conf_sigmod_heimelkm15_b200")

N, D = 1 << 22, 10
STEPS, FREE = 200, 50
CAP = 1 << 16
K_INIT = 0.0


@pytest.fixture(scope="module", autouse=True)
def _need_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    oracle.set_threads(0)


def _l1_slope(est_o, est_g, p):
    """L1 derivative sign(p_hat - p); ambiguous (p_hat within tolerance of p) -> the GPU's."""
    tol = 1e-7 + 1e-5 * abs(est_o)
    e = est_g if abs(est_o - p) <= tol else est_o
    return oracle.loss(oracle.LOSS_ABSOLUTE, 0.0, e, p)[1]


def _guard(Kv, tau, c, thr):
    amb = np.abs(Kv - tau) < 1e-6 / (N - 1) + 1e-9 * abs(tau)
    if np.isfinite(thr):
        amb |= np.abs(c - thr) < 1e-6 * thr
    return amb


def test_c5_full_size_stream_lockstep_and_free_running():
    import torch
    dev = torch.device("cuda")
    S0 = synth.make_data("gauss", N, D, seed=501)
    R = S0[synth.rng(501, 7).permutation(N)]                 # the database R (replacement pool)
    Q = synth.make_data("gauss", 1 << 16, D, seed=502)
    lo, hi = synth.workload(Q, STEPS, seed=503, kind="DT")
    dR = torch.from_numpy(R).to(dev)
    dlo, dhi = torch.from_numpy(lo).to(dev), torch.from_numpy(hi).to(dev)
    cnt = torch.zeros(STEPS, dtype=torch.int64, device=dev)
    K.kde_count_in_box_dev(dR, dlo, dhi, cnt)
    torch.cuda.synchronize()
    p = (cnt.double() / N).cpu().numpy()
    p[[7, 61, 133]] = 0.0                                     # true selectivity 0: eq. (20) at scale
    dp = torch.from_numpy(p).to(dev)
    tau = -1.0 / (N - 1)
    kp = K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=tau, k_max=4.0, k_init=K_INIT, empty_region=True)
    op = K.online_params(minibatch=10, loss=K.LOSS_ABSOLUTE, log_bandwidth=True)

    m = K.KDEModel.create(S0)
    m.set_retain(True)
    h0 = m.bandwidth
    d_idx = torch.zeros(CAP, dtype=torch.int64, device=dev)
    d_cnt = torch.zeros(1, dtype=torch.int64, device=dev)
    d_est = torch.zeros(1, dtype=torch.float64, device=dev)
    d_dpdh = torch.zeros(D, dtype=torch.float64, device=dev)
    npool = N - CAP

    S = S0.copy()                                             # host copy of the GPU sample
    Kg = np.zeros(N)
    st = oracle.OnlineState(D, lr0=op.lr0)
    # free-running oracle state
    S_f, h_f, K_f, st_f = S0.copy(), h0.copy(), np.zeros(N), oracle.OnlineState(D, lr0=op.lr0)
    free_ok = True
    total_amb = total_flag = n_empty_flags = 0
    for k in range(STEPS):
        h = m.bandwidth
        gs = m.online_state()
        off = (k * 977) % npool
        K.kde_stream_step_dev(m.handle, dlo[k:k + 1], dhi[k:k + 1], dp[k:k + 1], kp, op, d_idx, d_cnt,
                              dR[off:off + CAP], d_est, d_dpdh)
        torch.cuda.synchronize()
        est_g = float(d_est.item())
        g_g = d_dpdh.cpu().numpy()
        nf = int(d_cnt.item())
        idx_g = d_idx[:min(nf, CAP)].cpu().numpy()
        assert nf <= CAP and np.all(np.diff(idx_g) > 0)
        total_flag += nf

        # ---------------- lockstep: oracle from the GPU's pre-step state
        c_o = oracle.contributions(S, h, lo[k], hi[k])
        est_o, g_o = oracle.estimate_grad(S, h, lo[k:k + 1], hi[k:k + 1])
        assert abs(est_g - est_o[0]) <= 1e-7 + 1e-5 * abs(est_o[0]), (k, est_g, est_o[0])
        floor = 2.0 ** -60 / (np.sqrt(np.pi) * np.sqrt(np.log2(np.e)) * h)
        if not np.all(np.abs(g_g - g_o[0]) <= 1e-4 * np.abs(g_o[0]) + floor):  # m_j only when needed
            mabs = oracle.grad_abs_scale(S, h, lo[k:k + 1], hi[k:k + 1])[0]
            assert np.all(np.abs(g_g - g_o[0]) <= 1e-4 * np.abs(g_o[0]) + 1e-4 * mabs + floor), k
        thr = oracle.empty_region_threshold(h, lo[k], hi[k])[0] if p[k] == 0.0 else np.inf
        K_o = Kg.copy()
        idx_o = oracle.karma_update(c_o, est_o[0], p[k], oracle.LOSS_ABSOLUTE, 0.0, 4.0, tau, thr, K_o)
        amb = _guard(K_o, tau, c_o, thr)
        total_amb += int(amb.sum())
        fg = np.zeros(N, bool); fg[idx_g] = True
        fo = np.zeros(N, bool); fo[idx_o] = True
        assert nf == len(idx_g) or nf > CAP
        assert np.array_equal(fg[~amb], fo[~amb]), f"step {k}: flag sets differ"
        if p[k] == 0.0:
            n_empty_flags += nf                               # eq. (20) on a populated box
        # Listing 1 from the GPU's pre-step state
        if k > 0:  # the GPU's Listing 1 state is initialised (lr0) on first use
            st.acc, st.ms, st.lr, st.gprev, st.count = gs["acc"].copy(), gs["ms"].copy(), gs["lr"].copy(), \
                gs["gprev"].copy(), gs["count"]
        h_o = h.copy()
        oracle.online_step(st, h_o, _l1_slope(est_o[0], est_g, p[k]) * g_o[0] * h, batch=10, log_bw=True)
        h_g = m.bandwidth
        assert np.allclose(h_g, h_o, rtol=1e-4, atol=0), (k, h_g, h_o)
        # karma after the step: the update of eq. (8), then k_init on the replaced points
        K_o[idx_g] = K_INIT
        Kg_new = m.karma
        dK_scale = np.abs(K_o - Kg) + 1.0 / (N - 1)
        assert np.all(np.abs(Kg_new - K_o) <= 1e-4 * dK_scale + 1e-12), k
        Kg = Kg_new
        # the GPU replaced the flagged points (ascending) by the pool rows in order
        S[idx_g] = R[off:off + len(idx_g)]

        # ---------------- free-running oracle (first FREE queries)
        if k < FREE and free_ok:
            c_f = oracle.contributions(S_f, h_f, lo[k], hi[k])
            e_f, gr_f = oracle.estimate_grad(S_f, h_f, lo[k:k + 1], hi[k:k + 1])
            thr_f = oracle.empty_region_threshold(h_f, lo[k], hi[k])[0] if p[k] == 0.0 else np.inf
            Kf_pre = K_f
            K_f = K_f.copy()
            idx_f = oracle.karma_update(c_f, e_f[0], p[k], oracle.LOSS_ABSOLUTE, 0.0, 4.0, tau, thr_f, K_f)
            amb_f = _guard(K_f, tau, c_f, thr_f)
            ff = np.zeros(N, bool); ff[idx_f] = True
            assert np.array_equal(ff[~amb_f], fg[~amb_f]), f"free-running step {k}: flag sets differ"
            if amb_f[ff != fg].any():
                free_ok = False                               # an ambiguous flag: trajectories may part
            hf_pre = h_f.copy()
            oracle.online_step(st_f, h_f, _l1_slope(e_f[0], est_g, p[k]) * gr_f[0] * hf_pre, batch=10,
                               log_bw=True)
            assert np.allclose(h_g, h_f, rtol=1e-4, atol=0), (k, h_g, h_f)
            kk = idx_f[:CAP]
            K_f[kk] = K_INIT
            S_f[kk] = R[off:off + len(kk)]
            del Kf_pre

        if k in (0, 57, STEPS - 1):
            assert np.array_equal(m.sample, S), f"step {k}: host-tracked sample differs from the GPU's"
    assert total_flag > 0
    assert total_amb < 20
    print(f"c5 lockstep: {total_flag} flagged over {STEPS} steps ({n_empty_flags} by eq. 20), {total_amb} ambiguous")
