set -x
timeout 300 python -m pytest tests/test_gpu_cluster.py -x -q 2>&1 | tail -15
timeout 600 python -m pytest tests/test_gpu_l1.py tests/test_gpu_l0.py tests/test_gpu_dist.py tests/test_gpu_host.py -x -q 2>&1 | tail -15
timeout 600 python tools/scenarios.py "U:1024:1024:8" --opts '{"cluster_ctas":1}' 
timeout 600 python tools/scenarios.py "U:1024:1024:8" --opts '{"cluster_ctas":2}'
timeout 600 python tools/scenarios.py "U:1024:1024:8" --opts '{"cluster_ctas":4}'
timeout 600 python tools/scenarios.py "U:1024:1024:8" --opts '{"cluster_ctas":8}'
timeout 900 python tools/scenarios.py C5 "C5/8:0" "C5/4:0" "C5/2:0" "U:1024:1024:8" C3 C4 C2 --json gpurun_out/scen_r02b.json
