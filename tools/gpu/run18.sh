mkdir -p gpurun_out/r18
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r18/pytest_gpu.txt 2>&1; tail -3 gpurun_out/r18/pytest_gpu.txt
timeout 600 python bench.py > gpurun_out/r18/bench_c2.json 2> gpurun_out/r18/bench_c2.err; tail -c 400 gpurun_out/r18/bench_c2.json
for c in c3 c3s c3sg c5s c5; do timeout 900 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > gpurun_out/r18/bench_$c.json 2>&1; tail -1 gpurun_out/r18/bench_$c.json | cut -c1-120; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o gpurun_out/r18/prof_batched_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o gpurun_out/r18/prof_single_c3s python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r18/launches_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r18/launches_c3s.csv python bench.py --config c3s --steps 5 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r18/launches_c5.csv python bench.py --config c5 --steps 10 --warmup 3 --no-cpu > /dev/null 2>&1
ls gpurun_out/r18 | wc -l
