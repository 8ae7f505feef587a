"""Small run through every libkde entry point, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck) on the GPU box:

  compute-sanitizer --tool memcheck python tools/sanitize_run.py
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sigmod_heimelkm15_b200 as K  # noqa: E402
import synth  # noqa: E402


def run(d, n, q, kernel="gauss"):
    """q = 0: a batch of exactly 512 boxes (full 256-box CTAs: the culled batched scan)."""
    S = synth.make_data("gauss", n, d, seed=d)
    lo2, hi2 = synth.special_boxes(S, seed=d + 2)
    lo, hi = synth.mixed_workload(S, q if q else 512 - len(lo2), seed=d + 1)
    lo, hi = np.concatenate([lo, lo2]), np.concatenate([hi, hi2])
    p = synth.true_selectivity_cpu(S, lo, hi)
    m = K.KDEModel.create(S)
    if kernel == "epan":
        m.set_kernel("epan")
    m.set_retain(True)
    m.estimate(lo, hi, grad=True)
    m.estimate(lo, hi)
    for k in (0, 3, len(lo) - 1):
        m.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
        m.estimate(lo[k:k + 1], hi[k:k + 1])
    m.loss_and_grad(lo, hi, p, K.LOSS_RELATIVE, 1e-3, True)
    m.loss_and_grad(lo[:1], hi[:1], p[:1], K.LOSS_SQUARED_Q, 1e-3, False)
    kp = K.karma_params(threshold=-1.0 / (n - 1))
    idx, nf, _ = m.karma_update(lo[0], hi[0], 0.0, kp)
    m.online_update(lo[1], hi[1], p[1], K.online_params(minibatch=1))
    if nf:
        m.replace_points(idx, S[:nf][::-1].copy())
    dev = torch.device("cuda")
    dlo, dhi = torch.from_numpy(lo).to(dev), torch.from_numpy(hi).to(dev)
    dp = torch.from_numpy(p).to(dev)
    est = torch.zeros(len(lo), dtype=torch.float64, device=dev)
    g = torch.zeros((len(lo), d), dtype=torch.float64, device=dev)
    K.kde_estimate_batch_dev(m.handle, dlo[:1], dhi[:1], est[:1], g[:1])
    didx = torch.zeros(256, dtype=torch.int64, device=dev)
    dcnt = torch.zeros(1, dtype=torch.int64, device=dev)
    K.kde_karma_update_dev(m.handle, dlo[0], dhi[0], dp[:1], kp, didx, dcnt)
    K.kde_online_update_dev(m.handle, dp[:1], K.online_params(minibatch=1))
    rows = torch.from_numpy(S[:256].copy()).to(dev)
    K.kde_replace_points_dev(m.handle, didx, rows, dcnt)
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    K.kde_loss_and_grad_dev(m.handle, dlo, dhi, dp, loss, g[0], K.LOSS_ABSOLUTE, 0.0, False)
    torch.cuda.synchronize()
    cnt = torch.zeros(len(lo), dtype=torch.int64, device=dev)
    K.kde_count_in_box_dev(torch.from_numpy(S).to(dev), dlo, dhi, cnt)
    # device-resident streaming step (scan + cooperative karma / compaction / Listing 1 / replacement)
    fest = torch.zeros(1, dtype=torch.float64, device=dev)
    fg = torch.zeros(d, dtype=torch.float64, device=dev)
    for k in range(3):
        K.kde_stream_step_dev(m.handle, dlo[k:k + 1], dhi[k:k + 1], dp[k:k + 1], K.karma_params(threshold=0.0),
                              K.online_params(minibatch=2), didx, dcnt, rows, fest, fg)
    torch.cuda.synchronize()
    # reservoir inserts (host decision, accepted rows only)
    m.insert_rows(S[: min(n, 3000)][::-1].copy(), seed=5, n_seen=n)
    m.estimate(lo[:1], hi[:1], grad=True)
    # the ordered copy (cells.cu, scan_cells.cuh): rebuilt by this batch after the row changes above,
    # then single-box estimates without retained contributions read it too
    m.set_retain(False)
    m.estimate(lo, hi, grad=True)
    for k in (0, 3, len(lo) - 1):
        m.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
        m.estimate(lo[k:k + 1], hi[k:k + 1])
    K.kde_set_profiling(m.handle, True)                 # cells-scan counters
    m.estimate(lo, hi)
    m.estimate(lo[:1], hi[:1])
    K.kde_get_cells(m.handle, stats=True)
    K.kde_set_profiling(m.handle, False)
    torch.cuda.synchronize()
    m.close()


if __name__ == "__main__":
    for d, n, q, kern in [(3, 5003, 40, "gauss"), (10, 3001, 17, "gauss"), (13, 2053, 9, "gauss"),
                          (3, 9001, 0, "gauss"), (5, 4099, 0, "epan"), (10, 2051, 0, "gauss"),
                          (8, 20011, 0, "gauss"), (10, 40009, 33, "gauss"), (16, 9001, 5, "gauss")]:
        run(d, n, q, kern)
    print("sanitize run ok")
