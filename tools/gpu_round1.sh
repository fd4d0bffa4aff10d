#!/bin/bash
# first GPU check: smoke + parity (bounded), output under gpurun_out/
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/parity.log
tail -5 gpurun_out/smoke.log; tail -30 gpurun_out/parity.log
