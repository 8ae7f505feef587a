# batched scan: stage ring without CTA barriers (last warp out refills)
R=gpurun_out/r60; mkdir -p $R
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "c1 or dims or other or special or loss or c2_full or c3_full or mixed_narrow or small_batches or unbounded or offset or faces or bandwidth or epan or determinism" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for v in base minb3; do
  if [ $v = base ]; then unset KDE_LIB_PATH; else export KDE_LIB_PATH=$PWD/scratch/lib_$v.so; fi
  for c in c2 c3 c2e; do
    timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu > $R/bench_${v}_${c}.json 2>&1
    tail -1 $R/bench_${v}_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$v','$c', round(l['ms_per_step'],2), round(l['roofline']['frac'],3))" 2>&1 | tail -1
  done
done
unset KDE_LIB_PATH
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-cpu --no-cull > $R/bench_nocull_c2.json 2>&1; tail -1 $R/bench_nocull_c2.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('nocull c2', round(l['ms_per_step'],2), round(l['roofline']['frac'],3))"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > $R/ncu_c2.log 2>&1
