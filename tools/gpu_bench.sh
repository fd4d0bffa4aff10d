#!/bin/bash
# parity + bench + ncu evidence on one B200; everything lands in gpurun_out/
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu.txt 2>&1
timeout -s KILL 600 python -m pytest tests/ -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 2 gpurun_out/pytest_gpu.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -n 2 gpurun_out/smoke.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
# launch list of the headline command (cold-cache, serialised: shares, not absolutes)
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv \
   python bench.py --steps 3 --warmup 3 --no-others --no-cpu > gpurun_out/ncu_launch.log 2>&1; echo "launch rc=$?" >> gpurun_out/ncu_launch.log
for W in C5 C2 C3 C4 C1; do
  K=adiag; [ $W = C3 ] && K=fsk; [ $W = C4 ] && K=prevrow_cb
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 2 -c 1 \
     -o gpurun_out/prof_$W python tools/quick_time.py $W --reps 3 > gpurun_out/ncu_$W.log 2>&1
  echo "ncu $W rc=$?" >> gpurun_out/ncu_$W.log
done
head -c 1500 gpurun_out/bench.json; echo; tail -n 3 gpurun_out/bench.err
