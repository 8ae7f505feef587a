# Epanechnikov culling (single + batched) + batched cull tests
R=gpurun_out/r63; mkdir -p $R
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "cull or epan or mixed_narrow or c2_full or small_batches or determinism" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for c in c2e c3se; do
  for cl in "" "--no-cull"; do
    timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu $cl > $R/bench_${c}${cl}.json 2>&1
    tail -1 $R/bench_${c}${cl}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c $cl', round(l['ms_per_step'],4), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
