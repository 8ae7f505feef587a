mkdir -p gpurun_out/r13
timeout 1200 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/r13/sanitizer_synccheck.txt 2>&1; echo "synccheck rc=$?"; tail -2 gpurun_out/r13/sanitizer_synccheck.txt
timeout 1200 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/r13/sanitizer_racecheck.txt 2>&1; echo "racecheck rc=$?"; tail -2 gpurun_out/r13/sanitizer_racecheck.txt
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/r13/pytest_gpu.txt 2>&1; tail -2 gpurun_out/r13/pytest_gpu.txt
./tools/tune_batched | head -3
timeout 600 python bench.py --no-cpu --steps 10 > gpurun_out/r13/bench_c2.json 2>&1; tail -1 gpurun_out/r13/bench_c2.json | cut -c1-250
