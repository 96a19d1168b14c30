timeout 2400 python tools/autotune.py --out gpurun_out/autotune_r02b.json > gpurun_out/autotune_r02b.log 2>&1; tail -2 gpurun_out/autotune_r02b.log
