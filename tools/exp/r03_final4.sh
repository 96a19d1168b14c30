set -x
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_r02z4.log 2>&1; tail -3 gpurun_out/gpu_tests_r02z4.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02z4.log 2>&1; tail -1 gpurun_out/smoke_r02z4.log
timeout 900 python bench.py > gpurun_out/bench_r02z4_c5.json 2> gpurun_out/bench_r02z4_c5.err
for c in C1 C2 C3 C4; do timeout 900 python bench.py --config $c > gpurun_out/bench_r02z4_$c.json 2> gpurun_out/bench_r02z4_$c.err; done
timeout 900 python bench.py --impl reference > gpurun_out/bench_r02z4_reference.json 2> gpurun_out/bench_r02z4_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ncu_launches_r02z4_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launches_r02z4_c5.log 2>&1
