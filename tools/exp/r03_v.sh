timeout 1200 python -m pytest tests/test_gpu_l1.py -q 2>&1 | tail -3
