# UP (pairs per lane per step) sweep of the culled single-box scan + its parity tests
R=gpurun_out/r53; mkdir -p $R
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "cull or dims or c3_full or stream or karma or faces or c1" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for v in base up1t2k up2t2ko1 up2o1; do
  if [ $v = base ]; then unset KDE_LIB_PATH; else export KDE_LIB_PATH=$PWD/scratch/lib_$v.so; fi
  for c in c3s c3sg c5s; do
    timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $R/bench_${v}_${c}.json 2>&1
    tail -1 $R/bench_${v}_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$v','$c', round(l['ms_per_step']*1000,1), round(l['step_ms']['median']*1000,1), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
