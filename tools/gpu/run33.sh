# tuning sweep of the 2-point kernels (batched MINB/PU, single TILE/STAGES/OCC)
mkdir -p gpurun_out/r33
for v in base minb3 minb5 pu2 minb5pu2; do
  for cfg in "batched 3 1 1048576 10000 5" "batched 5 1 4194304 4096 3" "batched 3 1 1048576 100 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r33/kb.jsonl
  done
done
for v in base s512x3o4 s1024x3o3 s1024x2o3 s2048x2o2 s512x4o3; do
  for cfg in "single 5 0 16777216 20" "single 5 1 16777216 20" "single 3 1 16777216 20" "single 8 0 8388608 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r33/kb.jsonl
  done
done
