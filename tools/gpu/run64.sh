R=gpurun_out/r64; mkdir -p $R
for v in base m3 s2 s8; do
  if [ $v = base ]; then unset KDE_LIB_PATH; else export KDE_LIB_PATH=$PWD/scratch/lib_$v.so; fi
  for c in c2 c3 c2e; do
    timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu > $R/bench_${v}_${c}.json 2>&1
    tail -1 $R/bench_${v}_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$v','$c', round(l['ms_per_step'],2), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
