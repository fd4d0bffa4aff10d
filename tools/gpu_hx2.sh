export LDDP_TIMEOUT_MS=5000
for v in 2; do
LDDP_HX_VARIANT=$v timeout 300 python tools/hx_trace.py --cta 0 70 146 --debug 0 1 2 3
done > gpurun_out/hx_tr.log 2>&1
cat gpurun_out/hx_tr.log
