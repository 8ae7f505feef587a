mkdir -p gpurun_out/r5
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r5/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r5/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r5/smoke.txt 2>&1; tail -1 gpurun_out/r5/smoke.txt
timeout 600 python bench.py > gpurun_out/r5/bench_c2.json 2> gpurun_out/r5/bench_c2.err; tail -c 1500 gpurun_out/r5/bench_c2.json
for c in c3s c3sg c5s c3; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > gpurun_out/r5/bench_$c.json 2>&1; tail -1 gpurun_out/r5/bench_$c.json | cut -c1-300; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r5/launches_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/r5/ncu_launch_c2.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r5/launches_c3s.csv python bench.py --config c3s --steps 5 --warmup 3 --no-cpu > gpurun_out/r5/ncu_launch_c3s.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o gpurun_out/r5/prof_batched_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > gpurun_out/r5/ncu_full_batched.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o gpurun_out/r5/prof_single_c3s python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > gpurun_out/r5/ncu_full_single.log 2>&1
ls gpurun_out/r5
