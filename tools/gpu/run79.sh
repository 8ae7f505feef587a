R=gpurun_out/r79; mkdir -p $R
for b in scratch/kb/karma2_pb8_m4 scratch/kb/karma3_c8 scratch/kb/karma3_c5; do for n in 4194304 16777216; do echo -n "$b " >> $R/karma_ab.txt; timeout 60 $b $n 100 >> $R/karma_ab.txt 2>&1; done; done
cat $R/karma_ab.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -2 $R/pytest_gpu.txt
timeout 300 python bench.py --config c5 --steps 20 --warmup 3 > $R/bench_c5.json 2> $R/bench_c5.err; tail -c 600 $R/bench_c5.json
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c5.csv python bench.py --config c5 --steps 20 --warmup 3 > /dev/null 2>&1
