# compute-sanitizer over every entry point, now incl. the culled single-box and batched scans
R=gpurun_out/r68; mkdir -p $R
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool python tools/sanitize_run.py > $R/san_$tool.txt 2>&1
  echo "== $tool"; tail -2 $R/san_$tool.txt
done
