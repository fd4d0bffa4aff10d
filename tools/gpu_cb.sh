#!/bin/bash
# prev-row column-block kernel: parity + C4 sweep on one B200 (output under gpurun_out/)
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
timeout -s KILL 600 python -m pytest tests/test_gpu_prevrow_cb.py -x -q > gpurun_out/cb_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/cb_pytest.log
tail -n 15 gpurun_out/cb_pytest.log
timeout -s KILL 600 python tools/cb_sweep.py --variant 0 1 3 4 5 --warps 1 2 4 --reps 5 > gpurun_out/cb_sweep.log 2>&1
cut -c1-200 gpurun_out/cb_sweep.log
