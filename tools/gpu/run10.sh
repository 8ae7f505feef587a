mkdir -p gpurun_out/r10
./tools/tune_batched > gpurun_out/r10/tune_batched.jsonl; cat gpurun_out/r10/tune_batched.jsonl
timeout 900 python -m pytest tests/test_optimize.py -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/r10/pytest_opt.txt 2>&1; tail -5 gpurun_out/r10/pytest_opt.txt
