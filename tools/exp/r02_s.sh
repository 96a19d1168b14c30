timeout 900 python -m pytest tests/test_gpu_l1.py -x -q -k "panel" 2>&1 | tail -3
timeout 2400 python tools/autotune.py --cands panel_w16 --merge profiles/autotune_r02.json --out gpurun_out/autotune_r02c.json > gpurun_out/autotune_r02c.log 2>&1; tail -1 gpurun_out/autotune_r02c.log | cut -c1-200
