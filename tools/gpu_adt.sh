#!/bin/bash
export LDDP_TIMEOUT_MS=10000
timeout -s KILL 600 python -m pytest tests/test_gpu_adiag.py -x -q 2>&1 | tail -2
for spec in "C1 --rows 2" "C2 --rows 4" "C5 --rows 6"; do timeout -s KILL 300 python tools/ad_trace.py $spec 2>&1 | grep -E "normal ms|no-handoff|wait top"; done
