#!/bin/bash
export LDDP_TIMEOUT_MS=10000
timeout -s KILL 600 python -m pytest tests/test_gpu_adiag.py -x -q 2>&1 | tail -2
for D in 0 1 2 4 6; do
  LDDP_DEBUG=$D timeout -s KILL 200 python tools/quick_time.py C5 --rows 6 --reps 2 2>&1 | grep -v "^#" | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('debug $D', d.get('ms'), d.get('error',''))
"
done
for W in 4 8 16; do for R in 1 2 3 4 6; do LDDP_AD_W=$W timeout -s KILL 200 python tools/quick_time.py C5 --rows $R --reps 2 2>&1 | grep -v "^#" | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l)
    if 'error' in d: continue
    pl=d['plan']; print('C5 W',pl['warps'],'R',pl['rows_per_lane'],'E',pl['extra_lag'],'ms',d['ms'],'gcups',d['gcups'],'ok',d['parity'])
"; done; done
