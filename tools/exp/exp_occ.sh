for c in 1 0 2; do
  if [ $c = 1 ]; then L=""; else L="bash tools/exp/swap_run.sh tools/exp/libwcsvd_tp$c.so"; fi
  echo "cfg $c"; $L python tools/exp/occ.py
done
