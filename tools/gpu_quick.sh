#!/bin/bash
mkdir -p gpurun_out; rm -f gpurun_out/quick.jsonl
export LDDP_TIMEOUT_MS=20000
timeout -s KILL 300 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/parity_quick.log 2>&1; echo "parity rc=$?" >> gpurun_out/parity_quick.log
tail -3 gpurun_out/parity_quick.log
for spec in "C1 --variant 0 1 2 3" "C2 --variant 0 1 2 3" "C5 --variant 0 1 2 3" "C3 --rows 1 2"; do
  timeout -s KILL 300 python tools/quick_time.py $spec --reps 5 2>&1 | grep -v "^#" | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()); continue
    print(d.get('cfg'), 'var',d.get('variant'),'rows',d.get('rows'), 'ms',d.get('ms'), 'gcups',d.get('gcups'), 'ok',d.get('parity'), d.get('error',''))
" | tee -a gpurun_out/quick.txt
done
