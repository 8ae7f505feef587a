mkdir -p gpurun_out/r20
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r20/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r20/pytest_gpu.txt
timeout 900 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu > gpurun_out/r20/bench_c5.json 2>&1; tail -1 gpurun_out/r20/bench_c5.json | cut -c1-200
timeout 900 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu --no-graph > gpurun_out/r20/bench_c5_nograph.json 2>&1; tail -1 gpurun_out/r20/bench_c5_nograph.json | cut -c1-200
timeout 1500 python bench.py --config c4 --steps 3 --warmup 3 --no-cpu > gpurun_out/r20/bench_c4.json 2>&1; tail -1 gpurun_out/r20/bench_c4.json | cut -c1-300
