mkdir -p gpurun_out/r36
for v in base s1024x2o4 s2048x2o4 s1024x3o4 nobar nobar_o4; do
  for cfg in "single 5 0 16777216 20" "single 5 1 16777216 20" "single 3 1 16777216 20" "single 8 0 8388608 20" "single 8 1 8388608 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r36/kb.jsonl
  done
done
