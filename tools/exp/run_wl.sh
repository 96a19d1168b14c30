set -x
mkdir -p gpurun_out
cp paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so /tmp/main.so
cp tools/exp/libwcsvd_wl.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so
timeout 600 python -m pytest tests/test_gpu_l0.py tests/test_gpu_fp32.py tests/test_gpu_modes.py -x -q > gpurun_out/wl_tests.log 2>&1; echo "rc=$?" >> gpurun_out/wl_tests.log
tail -15 gpurun_out/wl_tests.log
for i in 1 2; do timeout 300 python tools/quick_time.py C2 2>&1 | tail -1; done
cp /tmp/main.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so
for i in 1 2; do timeout 300 python tools/quick_time.py C2 2>&1 | tail -1; done
