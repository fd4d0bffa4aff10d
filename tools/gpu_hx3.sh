export LDDP_TIMEOUT_MS=30000
O=gpurun_out/hx
mkdir -p $O
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:prevrow_hx -s 3 -c 1 \
  -o $O/prof_c4_hx -f python bench.py --workload C4 --no-others --no-cpu --steps 1 --warmup 3 > $O/ncu.log 2>&1
echo rc=$?
tail -3 $O/ncu.log
python tools/ncu_hot.py $O/prof_c4_hx.ncu-rep --top 60 > $O/hot.txt 2>&1
python tools/ncu_summary.py $O/prof_c4_hx.ncu-rep > $O/sum.json 2>&1
head -120 $O/hot.txt
cat $O/sum.json
