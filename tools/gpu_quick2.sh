#!/bin/bash
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
timeout -s KILL 300 python tools/quick_time.py C2 C5 C1 --reps 5 | cut -c1-400
timeout -s KILL 300 python tools/ad_sweep.py --cfg C2 --geoms 4,2,4 4,3,4 4,4,4 6,2,4 2,3,8 3,2,8 --reps 5 | cut -c1-90
timeout -s KILL 300 python tools/ad_sweep.py --cfg C5 --geoms 6,2,4 8,2,4 6,3,4 --reps 5 | cut -c1-90
