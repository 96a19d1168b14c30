for i in 1 2; do
timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-110
WCSVD_SLOTS_ALL=1 timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-110
WCSVD_PKG_DIR=tools/exp/old_pkg timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-110
done
nvidia-smi --query-gpu=clocks.sm,power.draw --format=csv
