R=gpurun_out/r80; mkdir -p $R
for i in 1 2 3; do for v in cur cm1 cm1km1; do
KDE_LIB_PATH=scratch/lib_$v.so timeout 300 python bench.py --config c5 --steps 50 --warmup 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['ms_per_step'], d['step_ms']['median'], d['e2e']['value'])" >> $R/ab.txt
done; done
cat $R/ab.txt
