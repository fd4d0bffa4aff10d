mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "diagmaxplus or invl or inverted" 2>&1 | tail -3 > gpurun_out/c6_pytest.log
timeout 300 python bench.py --workload C6 --steps 5 --warmup 3 --no-others --no-cpu > gpurun_out/c6.json 2>&1
