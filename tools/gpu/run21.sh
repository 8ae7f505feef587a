mkdir -p gpurun_out/r21
./tools/tune_batched > gpurun_out/r21/tune.jsonl 2>&1; head -12 gpurun_out/r21/tune.jsonl
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r21/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r21/pytest_gpu.txt
