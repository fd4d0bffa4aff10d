#!/bin/bash
# anti-diagonal geometry sweep on C5 / C2 / C1 (output under gpurun_out/)
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
timeout -s KILL 300 python tools/ad_sweep.py --cfg C5 --geoms 6,2,4 6,1,4 4,1,4 8,1,4 4,2,4 8,2,4 3,1,8 4,1,8 3,2,8 > gpurun_out/ad_sweep_c5.log 2>&1
timeout -s KILL 300 python tools/ad_sweep.py --cfg C2 --geoms 4,3,4 4,2,4 6,2,4 6,3,4 3,2,8 3,3,8 > gpurun_out/ad_sweep_c2.log 2>&1
timeout -s KILL 300 python tools/ad_sweep.py --cfg C1 --geoms 8,2,4 4,2,4 4,1,4 6,1,4 8,1,4 4,1,8 > gpurun_out/ad_sweep_c1.log 2>&1
cut -c1-100 gpurun_out/ad_sweep_c*.log
