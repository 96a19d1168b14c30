timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_r02t.log 2>&1; tail -3 gpurun_out/gpu_tests_r02t.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_r02t_c5.json 2> gpurun_out/bench_r02t_c5.err; tail -c 300 gpurun_out/bench_r02t_c5.json
timeout 600 python tools/scenarios.py "C5/8:0" "C5/4:0" "C5/2:0" C3 C4 "U:1024:1024:8" --json gpurun_out/scen_r02t.json 2>&1 | cut -c1-150
