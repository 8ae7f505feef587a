# culled single-box scan: tile / stages / occupancy sweep on the bench workloads
R=gpurun_out/r51; mkdir -p $R
for v in base o1 t1k t1ks3 t512 d10t2k d10t512o2; do
  if [ $v = base ]; then unset KDE_LIB_PATH; else export KDE_LIB_PATH=$PWD/scratch/lib_$v.so; fi
  for c in c3s c3sg c5s; do
    timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $R/bench_${v}_${c}.json 2>&1
    tail -1 $R/bench_${v}_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$v','$c', round(l['ms_per_step']*1000,1), l['step_ms'], round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
