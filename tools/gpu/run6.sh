mkdir -p gpurun_out/r6
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r6/pytest_gpu.txt 2>&1; tail -15 gpurun_out/r6/pytest_gpu.txt
timeout 600 python bench.py > gpurun_out/r6/bench_c2.json 2> gpurun_out/r6/bench_c2.err; tail -c 600 gpurun_out/r6/bench_c2.json
for c in c5 c3s c5s; do timeout 600 python bench.py --config $c --steps 50 --warmup 5 --no-cpu > gpurun_out/r6/bench_$c.json 2>&1; tail -3 gpurun_out/r6/bench_$c.json | cut -c1-400; done
