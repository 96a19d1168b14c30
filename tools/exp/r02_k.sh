timeout 900 python -m pytest tests/test_gpu_fp32.py tests/test_gpu_modes.py tests/test_gpu_host.py -x -q 2>&1 | tail -3
