mkdir -p gpurun_out/r34
for v in base s2048x2o2 s2048x2o3 s4096x2o1 s2048x3o2 reg2 reg4 reg2pf; do
  for cfg in "single 5 0 16777216 20" "single 5 1 16777216 20" "single 3 1 16777216 20" "single 8 0 8388608 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r34/kb.jsonl
  done
done
