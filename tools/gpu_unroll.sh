#!/bin/bash
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
for U in "" _u2 _u4; do
  echo "LIB=liblddp$U.so"
  LDDP_LIB_PATH=$PWD/paper_conf_ipps_kumark15_b200/liblddp$U.so timeout -s KILL 300 python tools/ad_sweep.py --cfg C5 --geoms 6,2,4 4,2,4 8,2,4 --reps 5 | cut -c1-90
  LDDP_LIB_PATH=$PWD/paper_conf_ipps_kumark15_b200/liblddp$U.so timeout -s KILL 300 python tools/ad_sweep.py --cfg C2 --geoms 4,2,4 --reps 5 | cut -c1-90
done
