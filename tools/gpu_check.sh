#!/bin/bash
# parity + default bench on one B200 (development check); output under gpurun_out/
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu.txt 2>&1
timeout -s KILL 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 2 gpurun_out/pytest_gpu.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
python - <<'P'
import json
d=json.loads(open('gpurun_out/bench.json').read().strip().splitlines()[-1])
print('C5', d['value'], d['ms_per_step'], d['roofline']['frac'])
for k,v in d.get('configs',{}).items(): print(k, v['value'], v['ms_per_step'], v['roofline']['frac'], v['parity']['match'])
P
