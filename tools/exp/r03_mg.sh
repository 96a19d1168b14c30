timeout 600 python -m pytest tests/test_gpu_l1.py -q -k "1024" 2>&1 | tail -2
timeout 600 python bench.py --gpus 2 --config C3 --batch 400 --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_gpus2.json 2> gpurun_out/bench_gpus2.err; echo rc=$?; tail -c 700 gpurun_out/bench_gpus2.json; tail -5 gpurun_out/bench_gpus2.err
