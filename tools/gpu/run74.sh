R=gpurun_out/r74; mkdir -p $R
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $R/smoke.txt 2>&1; tail -2 $R/smoke.txt
timeout 900 python bench.py > $R/bench_default.json 2>&1; tail -1 $R/bench_default.json | python -c "import sys,json; l=json.loads(sys.stdin.read()); print('default', round(l['ms_per_step'],3), '%.3g'%l['value'], l['roofline']['frac'], l['cpu_baseline']['value'], l['e2e'], l['gpu_launches'], l['clocks'])"
timeout 600 python bench.py --impl reference > $R/bench_reference.json 2>&1; tail -1 $R/bench_reference.json | cut -c1-150
