# A/B: Newton-Schulz cleanup of J (default) vs none (-DWCSVD_L1_NS=0), C3/C4/C5 device time + L1 parity
mkdir -p gpurun_out
for c in C3 C4 C5; do
  echo "== $c NS=1"; timeout 300 python tools/quick_time.py $c 2>&1 | tail -2
  echo "== $c NS=0"; timeout 300 bash tools/exp/swap_time.sh tools/exp/libwcsvd_nons.so $c 2>&1 | tail -2
done
echo "== parity NS=0"; timeout 600 bash tools/exp/swap_run.sh tools/exp/libwcsvd_nons.so python -m pytest tests/test_gpu_l1.py tests/test_gpu_robust.py -q -x 2>&1 | tail -5
