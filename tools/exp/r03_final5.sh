timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_r02z5.log 2>&1; tail -2 gpurun_out/gpu_tests_r02z5.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02z5.log 2>&1; tail -1 gpurun_out/smoke_r02z5.log
timeout 900 python bench.py > gpurun_out/bench_r02z5_c5.json 2> gpurun_out/bench_r02z5_c5.err
for c in C1 C2; do timeout 900 python bench.py --config $c > gpurun_out/bench_r02z5_$c.json 2> gpurun_out/bench_r02z5_$c.err; done
