# round-1 final refresh: full GPU suite, every bench line, launch lists, ncu captures of the dominant kernels
R=gpurun_out/r71; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -2 $R/pytest_gpu.txt
timeout 600 python bench.py > $R/bench_c2.json 2>&1; tail -1 $R/bench_c2.json | cut -c1-200
for c in c3 c3s c3sg c4 c5 c5s c2e c3se; do
    timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step'],4), round(l['roofline']['frac'],3), l['clocks'])" 2>&1 | tail -1
done
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-cpu --no-cull > $R/bench_c2_nocull.json 2>&1
timeout 300 python bench.py --config c3s --steps 20 --warmup 3 --no-cpu --no-cull > $R/bench_c3s_nocull.json 2>&1
timeout 300 python bench.py --impl reference > $R/bench_reference.json 2>&1; tail -1 $R/bench_reference.json | cut -c1-120
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c3s.csv python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c5.csv python bench.py --config c5 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c3s python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_c2e python bench.py --config c2e --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c3se python bench.py --config c3se --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
ls $R
