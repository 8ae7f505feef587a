R=gpurun_out/r82; mkdir -p $R
for i in 1 2; do for v in 2048 4096 8192; do for n in 4194304 16777216; do echo -n "pts$v " >> $R/karma_ab.txt; timeout 60 scratch/kb/karma4_p$v $n 100 >> $R/karma_ab.txt 2>&1; done; done; done
cat $R/karma_ab.txt
