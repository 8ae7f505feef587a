R=gpurun_out/r59; mkdir -p $R
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > $R/ncu_c2.log 2>&1
