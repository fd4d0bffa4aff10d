export LDDP_TIMEOUT_MS=5000
timeout 600 python -m pytest tests/test_gpu_prevrow_hx.py -x -q > gpurun_out/hx_t.log 2>&1; tail -3 gpurun_out/hx_t.log
timeout 300 python tools/quick_time.py C4 C7 --env LDDP_HX_VARIANT=${VARS:-0,2,6,8} --reps 5 > gpurun_out/hx_q.log 2>&1; grep -v '^#' gpurun_out/hx_q.log | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()[:300]); continue
    print(d.get('env'), d['cfg'], d.get('ms'), d.get('gcups'), d.get('parity'), d.get('plan',{}).get('kernel'), d.get('error','')[:200])"
LDDP_HX_VARIANT=0 timeout 300 python tools/hx_trace.py --cta 70 --debug 0 1 3 > gpurun_out/hx_tr.log 2>&1; cat gpurun_out/hx_tr.log
