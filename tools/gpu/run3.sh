mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu3.txt 2>&1; tail -25 gpurun_out/pytest_gpu3.txt
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench3_c2.txt 2>&1; tail -2 gpurun_out/bench3_c2.txt
timeout 600 python bench.py --config c3s --steps 50 --warmup 5 --no-cpu > gpurun_out/bench3_c3s.txt 2>&1; tail -2 gpurun_out/bench3_c3s.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o gpurun_out/prof3_single python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu3_single.log 2>&1; tail -2 gpurun_out/ncu3_single.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o gpurun_out/prof3_batched python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > gpurun_out/ncu3_batched.log 2>&1; tail -2 gpurun_out/ncu3_batched.log
