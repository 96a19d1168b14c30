timeout 900 python -m pytest tests/test_gpu_l0.py tests/test_gpu_modes.py tests/test_gpu_fp32.py tests/test_gpu_host.py tests/test_gpu_robust.py tests/test_gpu_dist.py -x -q 2>&1 | tail -4
for i in 1 2; do
WCSVD_LIBRARY=tools/exp/lib_head.so timeout 300 python tools/scenarios.py C1 "U:24:20:100" "U:32:32:2000" 2>&1 | cut -c1-110
timeout 300 python tools/scenarios.py C1 "U:24:20:100" "U:32:32:2000" 2>&1 | cut -c1-110
done
timeout 600 python bench.py --config C1 > gpurun_out/bench_r03r_C1.json 2>gpurun_out/bench_r03r_C1.err; tail -c 300 gpurun_out/bench_r03r_C1.json
