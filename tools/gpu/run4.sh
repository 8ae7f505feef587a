mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu4.txt 2>&1; tail -8 gpurun_out/pytest_gpu4.txt
for c in c2 c3s c3sg c5s c3; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > gpurun_out/bench4_$c.txt 2>&1; tail -1 gpurun_out/bench4_$c.txt | cut -c1-600; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o gpurun_out/prof4_batched python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu4_batched.log 2>&1; tail -1 gpurun_out/ncu4_batched.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o gpurun_out/prof4_single python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu4_single.log 2>&1; tail -1 gpurun_out/ncu4_single.log
