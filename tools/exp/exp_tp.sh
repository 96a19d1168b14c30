mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_l0.py tests/test_gpu_modes.py tests/test_gpu_fp32.py -x -q > gpurun_out/tp_tests.log 2>&1; echo rc=$? >> gpurun_out/tp_tests.log
python tools/quick_time.py C2 > gpurun_out/qt_tp_c2.txt 2>&1
python tools/quick_time.py C1 > gpurun_out/qt_tp_c1.txt 2>&1
python tools/quick_time.py C2 10000 '{"compute_uv": false}' > gpurun_out/qt_tp_c2_nouv.txt 2>&1
