timeout 900 python -m pytest tests/test_gpu_l1.py tests/test_gpu_cluster.py tests/test_gpu_robust.py -x -q 2>&1 | tail -2
for i in 1 2; do
timeout 600 python tools/scenarios.py C3 C4 --opts '{"_v":"full"}' | cut -c1-120
WCSVD_LIBRARY=tools/exp/lib_evdtri.so timeout 600 python tools/scenarios.py C3 C4 --opts '{"_v":"tri"}' | cut -c1-120
done
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C3 592
timeout 600 python tools/scenarios.py C5 | cut -c1-120
