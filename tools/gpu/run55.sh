# culled scan v2 (entry ring, gathers from the TMA stages): parity subset + sweep
R=gpurun_out/r55; mkdir -p $R
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "cull or dims or c3_full or stream or karma or faces" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for v in base s2 t2k o3; do
  if [ $v = base ]; then unset KDE_LIB_PATH; else export KDE_LIB_PATH=$PWD/scratch/lib_$v.so; fi
  for c in c3s c3sg c5s; do
    timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $R/bench_${v}_${c}.json 2>&1
    tail -1 $R/bench_${v}_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$v','$c', round(l['ms_per_step']*1000,1), round(l['step_ms']['median']*1000,1), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
unset KDE_LIB_PATH
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c3s python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > $R/ncu_c3s.log 2>&1
