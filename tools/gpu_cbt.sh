#!/bin/bash
# prev-row column-block: per-band trace of edge / interior blocks for several geometries
for V in ${VARS:-5}; do
LDDP_CB_VARIANT=$V timeout 300 python tools/cb_trace.py --block ${BLOCKS:-0 100} | sed "s/^/V=$V /"
done > gpurun_out/cbtrace3.log 2>&1
