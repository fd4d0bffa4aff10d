#!/bin/bash
# ncu --set full of the prev-row column-block kernel on C4 (output under gpurun_out/)
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
V=${V:-0}; NW=${NW:-2}
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:prevrow_cb -s 3 -c 1 \
   -o gpurun_out/prof_cb_v${V}_w${NW} python tools/cb_sweep.py --variant $V --warps $NW --reps 1 > gpurun_out/ncu_cb.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_cb.log
