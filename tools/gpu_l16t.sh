mkdir -p gpurun_out
for PE in "4 2" "6 2" "3 2"; do set -- $PE
LDDP_L16_P=$1 LDDP_L16_E=$2 timeout 300 python bench.py --workload C5 --steps 5 --warmup 3 --no-others --no-cpu > gpurun_out/l16_c5_$1$2.json 2>&1
done
LDDP_DEBUG=2 timeout 300 python tools/l16_trace.py --cfg C5 --out gpurun_out/l16_nohand.npy > gpurun_out/l16_nohand.json 2>&1
timeout 600 python -m pytest tests/test_gpu_lcs16.py -x -q 2>&1 | tail -3 > gpurun_out/l16_pytest.log
