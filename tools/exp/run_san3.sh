timeout 1500 python -m pytest tests/test_gpu_sanitizers.py -q --durations=0 2>&1 | tail -16
