#!/bin/bash
# fsk: per-step cost and lag (fs_scan) for several W:R:E settings in $RES
for RE in ${RES:-1:1:1}; do
  IFS=: read W R E <<< "$RE"
  LDDP_FSK_W=$W LDDP_FSK_R=$R LDDP_FSK_E=$E timeout 300 python tools/fs_scan.py --W 8192 --H 128 1024 8192 | sed "s/^/W=$W R=$R E=$E /"
done > gpurun_out/fss.log 2>&1
