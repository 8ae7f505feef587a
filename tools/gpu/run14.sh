mkdir -p gpurun_out/r14
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r14/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r14/pytest_gpu.txt
timeout 600 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu > gpurun_out/r14/bench_c5.json 2>&1; tail -1 gpurun_out/r14/bench_c5.json | cut -c1-250
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r14/launches_c5.csv python bench.py --config c5 --steps 10 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 1200 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/r14/racecheck.txt 2>&1; tail -1 gpurun_out/r14/racecheck.txt
