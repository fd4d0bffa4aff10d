mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_twins.py tests/test_gpu_abi.py -x -q 2>&1 | tail -15 > gpurun_out/twins_pytest.log
