mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_user_f.py tests/test_user_f_host.py -x -q 2>&1 | tail -15 > gpurun_out/userf_pytest.log
