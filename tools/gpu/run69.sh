R=gpurun_out/r69; mkdir -p $R
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"karma_kernel|compact_fused" -s 10 -c 2 -o $R/prof_c5k python bench.py --config c5 --steps 3 --warmup 3 --no-cpu --no-graph > $R/ncu.log 2>&1
tail -3 $R/ncu.log
