#!/bin/bash
# ncu --set full of the C1 and C2 wavefront kernels (development profiles)
mkdir -p gpurun_out
timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:wavefront -s 2 -c 1 \
   -o gpurun_out/prof_c1_v2 python tools/quick_time.py C1 --reps 3 > gpurun_out/ncu_c1.log 2>&1
timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:wavefront -s 2 -c 1 \
   -o gpurun_out/prof_c2_v2 python tools/quick_time.py C2 --reps 3 > gpurun_out/ncu_c2.log 2>&1
tail -n 3 gpurun_out/ncu_c1.log gpurun_out/ncu_c2.log
