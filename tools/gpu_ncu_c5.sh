#!/bin/bash
# ncu --set full (with source) of the C5 anti-diagonal kernel (output under gpurun_out/)
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
CFG=${CFG:-C5}
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:adiag -s 2 -c 1 \
   -o gpurun_out/prof_ad_${CFG} python tools/quick_time.py $CFG --reps 1 > gpurun_out/ncu_ad_${CFG}.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_ad_${CFG}.log
