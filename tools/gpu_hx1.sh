export LDDP_TIMEOUT_MS=5000
timeout 600 python -m pytest tests/test_gpu_prevrow_hx.py -x -q > gpurun_out/hx_t.log 2>&1; tail -15 gpurun_out/hx_t.log
timeout 300 python tools/quick_time.py C4 C7 --env LDDP_HX_VARIANT=-1,0,2,6,8 --reps 5 > gpurun_out/hx_q.log 2>&1; grep -v '^#' gpurun_out/hx_q.log | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()[:300]); continue
    print(d.get('env'), d['cfg'], d.get('ms'), d.get('gcups'), d.get('parity'), d.get('plan',{}).get('kernel'), d.get('error','')[:200])"
