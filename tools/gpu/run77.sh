R=gpurun_out/r77; mkdir -p $R
timeout 300 ncu --set full --import-source on --clock-control none -k regex:compact_fused -s 5 -c 1 -o $R/compact scratch/kb/karma_pb8_m4 4194304 10 > $R/ncu_compact.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:karma_kernel -s 5 -c 1 -o $R/karma scratch/kb/karma_pb8_m4 4194304 10 > $R/ncu_karma.log 2>&1
tail -3 $R/ncu_compact.log
