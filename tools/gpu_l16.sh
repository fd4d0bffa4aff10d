# lcs16 bring-up: parity tests, then C5 / C1 timings + trace (development script)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lcs16.py -x -q 2>&1 | tail -5 > gpurun_out/l16_pytest.log
for PE in "3 3" "3 4" "4 3" "2 3"; do set -- $PE
LDDP_L16_P=$1 LDDP_L16_E=$2 timeout 300 python bench.py --workload C5 --steps 5 --warmup 3 --no-others --no-cpu > gpurun_out/l16_c5_$1$2.json 2>&1
done
timeout 300 python bench.py --workload C1 --steps 20 --warmup 3 --no-others --no-cpu > gpurun_out/l16_c1.json 2>&1
timeout 300 python tools/l16_trace.py --cfg C5 > gpurun_out/l16_strips.json 2>&1
