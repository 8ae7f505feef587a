mkdir -p gpurun_out/r12
python tools/sanitize_run.py > gpurun_out/r12/plain.txt 2>&1; tail -1 gpurun_out/r12/plain.txt
for t in memcheck racecheck synccheck initcheck; do timeout 1200 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_run.py > gpurun_out/r12/sanitizer_$t.txt 2>&1; echo "== $t rc=$?"; tail -4 gpurun_out/r12/sanitizer_$t.txt; done
timeout 600 python -m pytest tests/test_c_example.py -m gpu -q -p no:cacheprovider > gpurun_out/r12/c_example.txt 2>&1; tail -2 gpurun_out/r12/c_example.txt
