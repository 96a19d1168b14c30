for k in 2 4; do echo "nstage $k"; for c in C3 C4; do timeout 300 bash tools/exp/swap_run.sh tools/exp/libwcsvd_ns$k.so python tools/quick_time.py $c 2>&1 | tail -1; done; done
echo "nstage 3"; for c in C3 C4; do timeout 300 python tools/quick_time.py $c 2>&1 | tail -1; done
