R=gpurun_out/r78; mkdir -p $R
for i in 1 2; do for b in scratch/kb/karma_pb8_m1 scratch/kb/karma_pb8_m4 scratch/kb/karma2_pb8_m1 scratch/kb/karma2_pb8_m4; do for n in 4194304 16777216; do echo -n "$b " >> $R/karma_ab.txt; timeout 60 $b $n 100 >> $R/karma_ab.txt 2>&1; done; done; done
cat $R/karma_ab.txt
