# round-1 refresh: full GPU suite, all bench lines, launch lists + ncu captures of the culled batched scan
R=gpurun_out/r62; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
timeout 600 python bench.py > $R/bench_c2.json 2>&1; tail -1 $R/bench_c2.json | cut -c1-300
for c in c3 c4 c2e c3se; do
    timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step'],3), round(l['roofline']['frac'],3))" 2>&1 | tail -1
done
timeout 300 python bench.py --impl reference > $R/bench_reference.json 2>&1; tail -1 $R/bench_reference.json | cut -c1-200
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_c3 python bench.py --config c3 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
