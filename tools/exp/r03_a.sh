nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_r03a_c5.json 2> gpurun_out/bench_r03a_c5.err; tail -c 400 gpurun_out/bench_r03a_c5.json
timeout 600 python tools/scenarios.py C2 C3 C4 --json gpurun_out/scen_r03a.json 2>&1 | cut -c1-150
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C3 592
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C4 592
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_r03a.log 2>&1; tail -3 gpurun_out/gpu_tests_r03a.log
