mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu2.txt 2>&1; tail -40 gpurun_out/pytest_gpu2.txt
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench2_c2.txt 2>&1; tail -2 gpurun_out/bench2_c2.txt
timeout 600 python bench.py --config c3s --steps 50 --warmup 5 --no-cpu > gpurun_out/bench2_c3s.txt 2>&1; tail -2 gpurun_out/bench2_c3s.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o gpurun_out/prof_single python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu_single.log 2>&1; tail -3 gpurun_out/ncu_single.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o gpurun_out/prof_batched python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu_batched.log 2>&1; tail -3 gpurun_out/ncu_batched.log
