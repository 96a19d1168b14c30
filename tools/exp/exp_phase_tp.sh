mkdir -p gpurun_out
bash tools/exp/swap_run.sh tools/exp/libwcsvd_phase.so python tools/exp/phase_tp.py C2 10000 > gpurun_out/phase_tp_c2.txt 2>&1
bash tools/exp/swap_run.sh tools/exp/libwcsvd_phase.so python tools/exp/phase_tp.py C2 10000 '{"compute_uv": false}' > gpurun_out/phase_tp_c2x.txt 2>&1
bash tools/exp/swap_run.sh tools/exp/libwcsvd_phase.so python tools/exp/phase_tp.py C2 1184 '{"compute_uv": false}' > gpurun_out/phase_tp_c2x_small.txt 2>&1
bash tools/exp/swap_run.sh tools/exp/libwcsvd_phase.so python tools/exp/phase_tp.py C2 148 '{"compute_uv": false}' > gpurun_out/phase_tp_c2x_1perSM.txt 2>&1
