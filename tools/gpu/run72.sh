R=gpurun_out/r72; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
for c in c2 c3s c2e; do
    timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step'],4), round(l['roofline']['frac'],3))" 2>&1 | tail -1
done
