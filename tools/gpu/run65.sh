R=gpurun_out/r65; mkdir -p $R
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "cull or epan or mixed_narrow or c2_full or c3_full or dims or special or unbounded" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for c in c2 c3 c2e c3s c3sg; do
    timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step'],4), round(l['roofline']['frac'],3))" 2>&1 | tail -1
done
