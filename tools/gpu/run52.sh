# ncu full captures of the culled single-box scan (c3s estimate, c5s d=10 grad+retain)
R=gpurun_out/r52; mkdir -p $R
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c5s python bench.py --config c5s --steps 2 --warmup 3 --no-cpu > $R/ncu_c5s.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c3s python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > $R/ncu_c3s.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 5 -c 1 -o $R/prof_c3sg python bench.py --config c3sg --steps 2 --warmup 3 --no-cpu > $R/ncu_c3sg.log 2>&1
ls -la $R
