R=gpurun_out/r67; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
python - > $R/smallq.txt 2>&1 <<'PY'
import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import synth, paper_conf_sigmod_heimelkm15_b200 as K
S = synth.make_data('gauss', 1 << 20, 3, seed=7)
m = K.KDEModel.create(S)
for q in (100, 300, 1000):
    lo, hi = synth.mixed_workload(S, q, seed=8)
    p = np.full(q, 0.01)
    for cull in (True, False):
        m.cull = cull
        for _ in range(3): m.loss_and_grad(lo, hi, p)
        torch.cuda.synchronize(); t0 = time.perf_counter()
        for _ in range(20): m.loss_and_grad(lo, hi, p)
        torch.cuda.synchronize(); print(q, cull, round((time.perf_counter() - t0) / 20 * 1e3, 3), 'ms')
PY
cat $R/smallq.txt
