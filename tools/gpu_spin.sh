#!/bin/bash
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
for S in 0 256 4096 100000; do
  echo "SPIN=$S"; LDDP_SPIN=$S timeout -s KILL 300 python tools/ad_sweep.py --cfg C5 --geoms 6,2,4 8,2,4 --reps 5 | cut -c1-90
  LDDP_SPIN=$S timeout -s KILL 300 python tools/ad_sweep.py --cfg C2 --geoms 4,2,4 --reps 5 | cut -c1-90
done
