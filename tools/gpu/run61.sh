# batched culling with the global probe order
R=gpurun_out/r61; mkdir -p $R
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "c1 or dims or other or special or loss or c2_full or c3_full or mixed_narrow or small_batches or unbounded or offset or faces or bandwidth or epan or determinism or shards" > $R/pytest.txt 2>&1; tail -2 $R/pytest.txt
for c in c2 c3 c4; do
    timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu > $R/bench_${c}.json 2>&1
    tail -1 $R/bench_${c}.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('$c', round(l['ms_per_step'],2), round(l['roofline']['frac'],3))" 2>&1 | tail -1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > $R/ncu_c2.log 2>&1
