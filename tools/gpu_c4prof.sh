#!/bin/bash
# ncu --set full of the prev-row column-block kernel on C4 for the variants in $VARS
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
for V in ${VARS:-5}; do
  LDDP_CB_VARIANT=$V timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:prevrow -s 3 -c 1 \
    -o gpurun_out/prof_c4_v$V -f python tools/cb_sweep.py --variant $V --warps 4 --reps 1 > gpurun_out/ncu_c4_v$V.log 2>&1
done
