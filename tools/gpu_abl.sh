#!/bin/bash
for X in 0 8 16; do
  L=$PWD/paper_conf_ipps_kumark15_b200/liblddp.so; [ $X != 0 ] && L=$PWD/paper_conf_ipps_kumark15_b200/liblddp_x$X.so
  echo "EXP=$X"; LDDP_LIB_PATH=$L LDDP_DEBUG=1 timeout 120 python tools/adiag_trace.py --cfg C5 2>&1 | grep -A5 "\"ms\"\|busy_cycles_per_step_by" | grep -v plan | head -8 | tr -d '\n'; echo
  LDDP_LIB_PATH=$L timeout 120 python tools/quick_time.py C5 C1 --reps 5 | cut -c1-110
done
