mkdir -p gpurun_out/r22
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r22/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r22/pytest_gpu.txt
for c in c2e c3se c2 c3s; do timeout 900 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > gpurun_out/r22/bench_$c.json 2>&1; tail -1 gpurun_out/r22/bench_$c.json | cut -c1-160; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o gpurun_out/r22/prof_single_c3se python bench.py --config c3se --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o gpurun_out/r22/prof_batched_c2e python bench.py --config c2e --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
