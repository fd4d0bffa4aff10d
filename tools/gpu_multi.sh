mkdir -p gpurun_out
python tools/dbg_multi.py > gpurun_out/dbg_multi.log 2>&1
timeout 900 python -m pytest tests/test_gpu_multi.py tests/test_gpu_watchdog.py tests/test_gpu_lcs16.py -x -q 2>&1 | tail -15 > gpurun_out/multi_pytest.log
