timeout 900 python -m pytest tests/test_gpu_l0.py tests/test_gpu_fp32.py tests/test_gpu_modes.py tests/test_gpu_host.py -q 2>&1 | tail -2
for i in 1 2 3; do WCSVD_LIBRARY=tools/exp/lib_pre.so timeout 300 python tools/scenarios.py C2 | cut -c1-120; timeout 300 python tools/scenarios.py C2 | cut -c1-120; done
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase_tp.py C2 10000 2>&1 | tail -7
