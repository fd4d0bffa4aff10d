#!/bin/bash
# C4 geometry sweep (cb_sweep) over $VARS
timeout 900 python tools/cb_sweep.py --variant ${VARS:-5} --warps ${WARPS:-4} --reps 5 > gpurun_out/cbsweep.log 2>&1
