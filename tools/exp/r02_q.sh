timeout 2400 python tools/autotune.py --out gpurun_out/autotune_r02.json > gpurun_out/autotune_r02.log 2>&1; tail -3 gpurun_out/autotune_r02.log
timeout 900 python bench.py > gpurun_out/bench_r02q_c5.json 2> gpurun_out/bench_r02q_c5.err; tail -c 600 gpurun_out/bench_r02q_c5.json
timeout 600 python bench.py --config C2 --no-cpu-baseline > gpurun_out/bench_r02q_c2.json 2>&1; tail -c 400 gpurun_out/bench_r02q_c2.json
