mkdir -p gpurun_out
python tools/quick_time.py C2 > gpurun_out/qt_c2_full.txt 2>&1
python tools/quick_time.py C2 10000 '{"compute_v": false}' > gpurun_out/qt_c2_nov.txt 2>&1
python tools/quick_time.py C2 10000 '{"compute_uv": false}' > gpurun_out/qt_c2_nouv.txt 2>&1
python tools/quick_time.py C2 10000 '{"force_path": 2}' > gpurun_out/qt_c2_l1.txt 2>&1
