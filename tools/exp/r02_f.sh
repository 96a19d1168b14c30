timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_r02f.log 2>&1; tail -3 gpurun_out/gpu_tests_r02f.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench_r02f_default.json 2> gpurun_out/bench_r02f_default.err; tail -c 3000 gpurun_out/bench_r02f_default.json; tail -5 gpurun_out/bench_r02f_default.err
timeout 900 python bench.py --gpus 2 --no-cpu-baseline --steps 2 --warmup 1 > gpurun_out/bench_r02f_g2.json 2> gpurun_out/bench_r02f_g2.err; tail -c 1500 gpurun_out/bench_r02f_g2.json; tail -5 gpurun_out/bench_r02f_g2.err
timeout 600 python bench.py --impl reference --steps 1 --warmup 1 > gpurun_out/bench_r02f_ref.json 2>&1; tail -c 1500 gpurun_out/bench_r02f_ref.json
