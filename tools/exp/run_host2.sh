export WCSVD_DEBUG=1
timeout 120 python tools/exp/dbg_host.py 3
timeout 120 python tools/exp/dbg_host.py 40
CUDA_LAUNCH_BLOCKING=1 timeout 300 python tools/exp/dbg_host.py 40
timeout 600 python bench.py --config C2 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bh_C2.json 2> gpurun_out/bh_C2.err; tail -c 400 gpurun_out/bh_C2.json; tail -5 gpurun_out/bh_C2.err
