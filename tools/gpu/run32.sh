# 2-point packed evaluation (point_box2): kbench + GPU parity
mkdir -p gpurun_out/r32
for v in pair; do
  for cfg in "batched 3 1 1048576 10000 5" "batched 3 1 1048576 100 20" "batched 5 1 4194304 4096 5" "batched 8 1 4194304 4096 3" "single 5 0 16777216 20" "single 5 1 16777216 20" "single 10 0 4194304 20" "single 10 1 4194304 20" "single 3 1 16777216 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r32/kb.jsonl
  done
done
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/r32/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r32/pytest_gpu.txt
