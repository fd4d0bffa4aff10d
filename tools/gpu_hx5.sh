export LDDP_TIMEOUT_MS=5000
for rep in 1 2; do
timeout 300 python tools/quick_time.py C4 C7 --env LDDP_HX_VARIANT=${VARS:--1,0,2,6} --reps 10 2>&1 | grep -v '^#' | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()[:300]); continue
    print(d.get('env'), d['cfg'], d.get('ms'), d.get('min'), d.get('parity'), d.get('plan',{}).get('kernel'))"
done
