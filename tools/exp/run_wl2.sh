set -x
echo WL; timeout 300 bash tools/exp/swap_run.sh tools/exp/libwcsvd_wl_phase.so python tools/exp/phase_tp.py C2 10000 2>&1 | tail -9
echo BASE; timeout 300 bash tools/exp/swap_run.sh tools/exp/libwcsvd_phase.so python tools/exp/phase_tp.py C2 10000 2>&1 | tail -9
