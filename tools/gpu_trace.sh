#!/bin/bash
# in-kernel globaltimer traces of small wavefront fills (development)
mkdir -p gpurun_out
export LDDP_TIMEOUT_MS=20000
timeout -s KILL 120 python tools/trace_run.py --func lcs --rows 1024 --cols 1024 --out gpurun_out/trace_c1.json > gpurun_out/trace_c1.log 2>&1
timeout -s KILL 120 python tools/trace_run.py --func lcs --rows 4096 --cols 8192 --out gpurun_out/trace_lcs4k.json > gpurun_out/trace_lcs4k.log 2>&1
head -60 gpurun_out/trace_c1.log
