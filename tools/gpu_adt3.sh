#!/bin/bash
export LDDP_TIMEOUT_MS=10000
for D in 2 4; do echo "== debug $D"; LDDP_DEBUG=$D timeout -s KILL 300 python tools/ad_trace.py C5 --rows 6 2>&1 | grep -v "^{" | head -16; done
