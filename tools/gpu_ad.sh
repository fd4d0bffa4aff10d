#!/bin/bash
# adiag kernel: parity + quick timings (development)
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=10000
timeout -s KILL 600 python -m pytest tests/test_gpu_adiag.py -x -q > gpurun_out/ad_parity.log 2>&1; echo "rc=$?" >> gpurun_out/ad_parity.log
tail -5 gpurun_out/ad_parity.log
for E in 2 3; do LDDP_AD_E=$E timeout -s KILL 300 python tools/quick_time.py C1 C2 --rows 2 3 4 6 --reps 5 2>&1 | grep -v "^#" | cut -c1-150; done
for W in 4 8; do LDDP_AD_W=$W timeout -s KILL 600 python tools/quick_time.py C5 --rows 3 4 6 --reps 3 2>&1 | grep -v "^#" | cut -c1-150; done
LDDP_AD_E=3 timeout -s KILL 600 python tools/quick_time.py C5 --rows 4 6 --reps 3 2>&1 | grep -v "^#" | cut -c1-150
