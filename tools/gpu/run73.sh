R=gpurun_out/r73; mkdir -p $R
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "karma or stream or replace or epan or cull or determinism or invalid" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
timeout 600 python tools/gpu/dbg_stream.py > $R/dbg.txt 2>&1; tail -2 $R/dbg.txt
for c in c5 c5s c3s; do
    timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step']*1000,1), round(l['roofline']['frac'],3), l.get('stream'))" 2>&1 | tail -1
done
timeout 300 python bench.py --config c5 --steps 30 --warmup 3 --no-cpu --no-graph > $R/bench_c5_nograph.json 2>&1; tail -1 $R/bench_c5_nograph.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('c5 nograph', round(l['ms_per_step']*1000,1))"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c5.csv python bench.py --config c5 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
