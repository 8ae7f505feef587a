# full GPU suite after the culled-scan v3 + noinline Listing 1 body; c2 / c3s / c5 bench lines
R=gpurun_out/r57; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
for c in c3s c3sg c5s c5; do
    timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step']*1000,1), round(l['step_ms']['median']*1000,1), round(l['roofline']['frac'],3))" 2>&1 | tail -1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c3s.csv python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c5.csv python bench.py --config c5 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c5s python bench.py --config c5s --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
