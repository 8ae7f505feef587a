mkdir -p gpurun_out/r24
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r24/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r24/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py > gpurun_out/r24/bench_c2.json 2> gpurun_out/r24/bench_c2.err; tail -c 300 gpurun_out/r24/bench_c2.json
for c in c3 c3s c3sg c5s c5 c2e c3se; do timeout 900 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > gpurun_out/r24/bench_$c.json 2>&1; tail -1 gpurun_out/r24/bench_$c.json | cut -c1-100; done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r24/bench_ref.json 2>&1; tail -1 gpurun_out/r24/bench_ref.json | cut -c1-200
