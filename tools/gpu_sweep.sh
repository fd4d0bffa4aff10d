#!/bin/bash
# geometry sweep of the adiag kernel vs the old wavefront kernel (development)
export LDDP_TIMEOUT_MS=10000
pj() { python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    if 'error' in d: continue
    pl=d['plan']; print(d['cfg'], pl['kernel'], 'W',pl['warps'],'R',pl['rows_per_lane'],'E',pl['extra_lag'],'ms',d['ms'],'gcups',d['gcups'],'ok',d['parity'])
"; }
for C in C1 C2; do LDDP_KERNEL=wavefront timeout -s KILL 200 python tools/quick_time.py $C --reps 3 2>&1 | pj; done
for W in 4 8; do for E in 2 3 4; do
  LDDP_AD_W=$W LDDP_AD_E=$E timeout -s KILL 300 python tools/quick_time.py C1 C2 --rows 2 3 4 6 --reps 3 2>&1 | pj
done; done
for W in 4 8; do for E in 2 3; do
  LDDP_AD_W=$W LDDP_AD_E=$E timeout -s KILL 300 python tools/quick_time.py C5 --rows 3 4 6 8 --reps 2 2>&1 | pj
done; done
