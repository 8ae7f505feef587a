# packed Epanechnikov (phi_epan2), face-ties test, graph warm-up fix in bench
R=gpurun_out/r41; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
for c in c2e c3se c5; do timeout 900 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > $R/bench_$c.json 2>&1; tail -1 $R/bench_$c.json | cut -c1-100; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_batched_c2e python bench.py --config c2e --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o $R/prof_single_c3se python bench.py --config c3se --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
