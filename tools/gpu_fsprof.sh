#!/bin/bash
# C3 (Floyd-Steinberg 8192^2, fsk): bench line, then ncu --set full of one fsk launch
mkdir -p gpurun_out
timeout 300 python bench.py --workload C3 --no-others --no-cpu --steps 10 --warmup 3 > gpurun_out/c3.json 2> gpurun_out/c3.err
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:fsk -s 3 -c 1 -o gpurun_out/prof_c3 -f \
  python bench.py --workload C3 --no-others --no-cpu --steps 2 --warmup 3 > gpurun_out/ncu_c3.log 2>&1
