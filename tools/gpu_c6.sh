#!/bin/bash
# C6 (inverted-L 32768^2): invl register-block depth sweep (LDDP_INVL_BLOCK), device-timed by bench.py
for B in ${BLKS:-16 32 48}; do
  LDDP_INVL_BLOCK=$B timeout 300 python bench.py --workload C6 --no-others --no-cpu --steps 10 --warmup 3 2>/dev/null | \
    python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('BLK', $B, d['ms_per_step'], d['value'], d['parity']['match'])"
done
