# phi v2 (K=6 full polynomial, clamp, pair RCP, fused bracket) vs v1: tuning sweeps + GPU parity
mkdir -p gpurun_out/r30
for v in v1 v2; do
  timeout 300 ./scratch/tune_single_$v > gpurun_out/r30/tune_single_$v.jsonl 2>&1
  timeout 300 ./scratch/tune_batched_$v > gpurun_out/r30/tune_batched_$v.jsonl 2>&1
done
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r30/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r30/pytest_gpu.txt
