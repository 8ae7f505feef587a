import sys, numpy as np, torch
sys.path.insert(0, '.')
import synth, paper_conf_sigmod_heimelkm15_b200 as K
def run(cull):
    n, d, steps, cap = 20000, 4, 24, 4096
    S = synth.make_data("gauss", n, d, seed=40)
    R = synth.make_data("gauss", 80000, d, seed=40)
    lo, hi = synth.workload(S, steps, seed=41, kind="DT")
    p = synth.true_selectivity_cpu(R, lo, hi); p[5] = 0.0
    pool = synth.replacement_rows(R, steps * cap, seed=42, step=0)
    kp = K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=-1.0 / (n - 1), k_max=4.0)
    op = K.online_params(minibatch=5, loss=K.LOSS_ABSOLUTE, log_bandwidth=True)
    mh, mf = K.KDEModel.create(S), K.KDEModel.create(S)
    for m in (mh, mf): m.set_retain(True); m.cull = cull
    dev = torch.device("cuda")
    dlo, dhi = torch.from_numpy(lo).to(dev), torch.from_numpy(hi).to(dev)
    dp = torch.from_numpy(p).to(dev); dpool = torch.from_numpy(pool).to(dev)
    fidx = torch.zeros(cap, dtype=torch.int64, device=dev); fcnt = torch.zeros(1, dtype=torch.int64, device=dev)
    fest = torch.zeros(1, dtype=torch.float64, device=dev); fdpdh = torch.zeros(d, dtype=torch.float64, device=dev)
    s = torch.cuda.current_stream()
    for k in range(steps):
        e_h, g_h = mh.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
        idx, nf, trunc = mh.karma_update(lo[k], hi[k], p[k], kp)
        st_h0 = mh.online_state()
        mh.online_update(lo[k], hi[k], p[k], op)
        mh.replace_points(idx, pool[k * cap:k * cap + len(idx)])
        st_f0 = mf.online_state()
        K.kde_stream_step_dev(mf.handle, dlo[k:k + 1], dhi[k:k + 1], dp[k:k + 1], kp, op, fidx, fcnt,
                              dpool[k * cap:(k + 1) * cap], fest, fdpdh, stream=s)
        torch.cuda.synchronize()
        ok = (fest.item() == e_h[0], np.array_equal(fdpdh.cpu().numpy(), g_h[0]), int(fcnt.item()) == nf,
              np.array_equal(mf.bandwidth, mh.bandwidth))
        print(cull, k, ok, nf, e_h[0], fest.item())
        if not all(ok):
            print(" h", mh.bandwidth - mf.bandwidth, "\n state_h0", st_h0, "\n state_f0", st_f0)
            print(" state_h1", mh.online_state(), "\n state_f1", mf.online_state())
            print(" grad", g_h[0], fdpdh.cpu().numpy())
            break
run(True); run(False)
