R=gpurun_out/r76; mkdir -p $R
for b in scratch/kb/karma_*; do for n in 4194304 16777216; do timeout 60 $b $n 50 >> $R/karma_ab.jsonl 2>&1; done; done
cat $R/karma_ab.jsonl
