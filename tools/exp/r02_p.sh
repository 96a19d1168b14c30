timeout 900 python -m pytest tests/test_gpu_l1.py tests/test_gpu_cluster.py -x -q 2>&1 | tail -2
for i in 1 2; do
timeout 600 python tools/scenarios.py C3 C4 --opts '{"_v":"new"}'
WCSVD_PKG_DIR=tools/exp/headpkg timeout 600 python tools/scenarios.py C3 C4 --opts '{"_v":"head"}'
done
