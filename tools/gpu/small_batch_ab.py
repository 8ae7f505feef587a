"""A/B of small batches (the ~100-box training sets of batch optimisation):
culled scan over the ordered copy vs the sample-order path (phase-split unculled batched scan)."""
import json, sys, time
import numpy as np
import torch
sys.path.insert(0, ".")
import synth
import paper_conf_sigmod_heimelkm15_b200 as K

S = synth.make_data("gauss", 1 << 24, 5, seed=7)
Q = synth.make_data("gauss", 1 << 16, 5, seed=7)
m = K.KDEModel.create(S)
out = {}
for q in (16, 100, 256, 1000):
    lo, hi = synth.mixed_workload(Q, q, 8)
    dlo, dhi = torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda()
    est = torch.zeros(q, dtype=torch.float64, device="cuda")
    g = torch.zeros((q, 5), dtype=torch.float64, device="cuda")
    for cells in (True, False):
        m.cells = cells
        for _ in range(3):
            K.kde_estimate_batch_dev(m.handle, dlo, dhi, est, g, stream=torch.cuda.current_stream())
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            K.kde_estimate_batch_dev(m.handle, dlo, dhi, est, g, stream=torch.cuda.current_stream())
        e1.record()
        torch.cuda.synchronize()
        out[f"q{q}_{'cells' if cells else 'unordered'}_ms"] = e0.elapsed_time(e1) / 10
print(json.dumps(out))
# sanity: wall-clock of one call and the estimates
lo, hi = synth.mixed_workload(Q, 1000, 8)
m.cells = True
torch.cuda.synchronize(); t0 = time.perf_counter()
e, gg = m.estimate(lo, hi, grad=True)
torch.cuda.synchronize()
print(json.dumps({"host_call_ms": (time.perf_counter() - t0) * 1e3, "est_mean": float(np.mean(e)), "est_max": float(np.max(e))}))
