mkdir -p gpurun_out/r7
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r7/pytest_gpu.txt 2>&1; tail -5 gpurun_out/r7/pytest_gpu.txt
for c in c3s c3sg c5s c5; do timeout 600 python bench.py --config $c --steps 50 --warmup 5 --no-cpu > gpurun_out/r7/bench_$c.json 2>&1; tail -1 gpurun_out/r7/bench_$c.json | cut -c1-200; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r7/launches_c5.csv python bench.py --config c5 --steps 10 --warmup 3 --no-cpu > gpurun_out/r7/ncu_launch_c5.log 2>&1
