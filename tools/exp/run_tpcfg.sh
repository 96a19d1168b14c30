for c in 1 2 3; do
  if [ $c = 3 ]; then L=tools/exp/libwcsvd_wl.so; else L=tools/exp/libwcsvd_tp$c.so; fi
  echo "cfg $c"; timeout 300 bash tools/exp/swap_run.sh $L python tools/quick_time.py C2 2>&1 | tail -1
done
echo "cfg 0"; timeout 300 python tools/quick_time.py C2 2>&1 | tail -1
