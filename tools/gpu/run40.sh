# round-1 refresh after the 2-point packed Phi + warp-specialised single scan
R=gpurun_out/r40; mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $R/pytest_gpu.txt 2>&1; tail -3 $R/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $R/smoke.txt 2>&1; tail -1 $R/smoke.txt
timeout 600 python bench.py > $R/bench_c2.json 2> $R/bench_c2.err; tail -c 300 $R/bench_c2.json
for c in c3 c3s c3sg c5s c5 c2e c3se; do timeout 900 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > $R/bench_$c.json 2>&1; tail -1 $R/bench_$c.json | cut -c1-100; done
timeout 1500 python bench.py --config c4 --steps 3 --warmup 3 --no-cpu > $R/bench_c4.json 2>&1; tail -1 $R/bench_c4.json | cut -c1-100
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $R/bench_ref.json 2>&1; tail -1 $R/bench_ref.json | cut -c1-100
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_batched -s 3 -c 1 -o $R/prof_batched_c2 python bench.py --config c2 --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_single -s 3 -c 1 -o $R/prof_single_c3s python bench.py --config c3s --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $R/launches_c3s.csv python bench.py --config c3s --steps 5 --warmup 3 --no-cpu > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $R/launches_c5.csv python bench.py --config c5 --steps 10 --warmup 3 --no-cpu > /dev/null 2>&1
for cfg in "batched 3 1 1048576 10000 5" "batched 5 1 4194304 4096 5" "batched 8 1 4194304 4096 3" "single 5 0 16777216 20" "single 5 1 16777216 20" "single 8 0 8388608 20" "single 8 1 8388608 20" "single 10 0 4194304 20" "single 10 1 4194304 20"; do
  timeout 120 ./scratch/kb_final $cfg >> $R/kbench.jsonl
done
ls $R | wc -l
