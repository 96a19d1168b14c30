timeout 900 python -m pytest tests/test_gpu_l1.py tests/test_gpu_robust.py tests/test_gpu_cluster.py -x -q 2>&1 | tail -4
timeout 600 python tools/robustness.py > gpurun_out/robust_r02m.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/robust_r02m.json')); print(json.dumps({k: v for k, v in d.items() if k != 'fig15'}, indent=0)[:3000])"
for i in 1 2; do
timeout 600 python tools/scenarios.py C3 C4 --opts '{"_v":"fast"}'
WCSVD_LIBRARY=tools/exp/lib_evd0.so timeout 600 python tools/scenarios.py C3 C4 --opts '{"_v":"evd0"}'
done
timeout 600 python tools/scenarios.py C5 --opts '{"_v":"fast"}'
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C3 592
