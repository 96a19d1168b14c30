set -x
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_r02z3.log 2>&1; tail -3 gpurun_out/gpu_tests_r02z3.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02z3.log 2>&1; tail -1 gpurun_out/smoke_r02z3.log
timeout 900 python bench.py > gpurun_out/bench_r02z3_c5.json 2> gpurun_out/bench_r02z3_c5.err; tail -c 200 gpurun_out/bench_r02z3_c5.json
timeout 900 python bench.py --config C2 > gpurun_out/bench_r02z3_C2.json 2> gpurun_out/bench_r02z3_C2.err
timeout 900 python bench.py --config C3 > gpurun_out/bench_r02z3_C3.json 2> gpurun_out/bench_r02z3_C3.err
