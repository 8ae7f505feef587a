# tail-culled single-box scan: GPU tests, A/B bench on the single-box configs
R=gpurun_out/r50; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
for c in c3s c3sg c5s c5; do
  for cl in "" "--no-cull"; do
    timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu $cl > $R/bench_${c}${cl}.json 2>&1
    tail -1 $R/bench_${c}${cl}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c','$cl', round(l['ms_per_step'],4), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
