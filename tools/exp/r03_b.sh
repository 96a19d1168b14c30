timeout 600 python tools/scenarios.py C2 C3 C4 --json gpurun_out/scen_r03b.json 2>&1 | cut -c1-150
WCSVD_LIBRARY=tools/exp/lib_rot32.so timeout 600 python tools/scenarios.py C3 C4 2>&1 | cut -c1-150
timeout 900 python -m pytest tests/test_gpu_l0.py tests/test_gpu_l1.py tests/test_gpu_host.py -x -q 2>&1 | tail -2
WCSVD_LIBRARY=tools/exp/lib_rot32.so timeout 900 python -m pytest tests/test_gpu_l1.py tests/test_gpu_robust.py -x -q 2>&1 | tail -2
WCSVD_LIBRARY=tools/exp/lib_rot32.so timeout 900 python tools/robustness.py > gpurun_out/robust_rot32.json 2>&1; tail -c 1500 gpurun_out/robust_rot32.json
