R=gpurun_out/r81; mkdir -p $R
for i in 1 2 3; do for v in intree cur; do
if [ $v = intree ]; then L=""; else L=scratch/lib_$v.so; fi
KDE_LIB_PATH=$L timeout 300 python bench.py --config c5 --steps 50 --warmup 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['ms_per_step'], d['step_ms']['median'], d['e2e']['value'])" >> $R/ab.txt
done; done
cat $R/ab.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -2 $R/pytest_gpu.txt
timeout 300 python bench.py --config c5 --steps 20 --warmup 3 > $R/bench_c5.json 2> $R/bench_c5.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c5.csv python bench.py --config c5 --steps 20 --warmup 3 > /dev/null 2>&1
timeout 300 python bench.py > $R/bench_default.json 2> $R/bench_default.err; tail -c 300 $R/bench_default.json
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
