#!/bin/bash
# usage: CFG=C5 LDDP_DEBUG=1 bash tools/gpu_ncu_ad.sh
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
CFG=${CFG:-C2}
LDDP_DEBUG=${LDDP_DEBUG:-0} timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:adiag -s 2 -c 1 \
   -o gpurun_out/prof_ad_${CFG}_d${LDDP_DEBUG:-0} python tools/quick_time.py $CFG --reps 2 > gpurun_out/ncu_ad_$CFG.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_ad_$CFG.log
