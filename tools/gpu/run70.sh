R=gpurun_out/r70; mkdir -p $R
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "cull or dims or stream or karma or c3_full" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for v in base pb16; do
  if [ $v = base ]; then unset KDE_LIB_PATH; else export KDE_LIB_PATH=$PWD/scratch/lib_$v.so; fi
  for c in c5s c5; do
    timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $R/bench_${v}_${c}.json 2>&1
    tail -1 $R/bench_${v}_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$v','$c', round(l['ms_per_step']*1000,1), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
