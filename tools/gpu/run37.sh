mkdir -p gpurun_out/r37
for v in base w1024x4o2 w2048x2o2 w2048x3o1 w512x4o3 w512x6o2 w1024x3o3; do
  for cfg in "single 5 0 16777216 20" "single 5 1 16777216 20" "single 3 1 16777216 20" "single 8 0 8388608 20" "single 8 1 8388608 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r37/kb.jsonl
  done
done
