# kbench variant sweep + ncu full captures of the base variant
mkdir -p gpurun_out/r31
for v in base nohs noclamp k5 k4; do
  for cfg in "batched 3 1 1048576 10000 5" "batched 5 1 4194304 4096 5" "single 5 0 16777216 20" "single 5 1 16777216 20" "single 10 0 4194304 20"; do
    timeout 120 ./scratch/kb_$v $cfg | sed "s/^{/{\"v\":\"$v\",/" >> gpurun_out/r31/kb.jsonl
  done
done
timeout 600 ncu --set full --import-source on -k regex:scan_batched -s 2 -c 1 -o gpurun_out/r31/batched_d3 ./scratch/kb_base batched 3 1 1048576 10000 1 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on -k regex:scan_single -s 2 -c 1 -o gpurun_out/r31/single_d5 ./scratch/kb_base single 5 0 16777216 1 > /dev/null 2>&1
ls gpurun_out/r31
