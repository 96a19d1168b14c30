WCSVD_LIBRARY=tools/exp/lib_pre.so python tools/exp/dump.py /tmp/a.npz | tail -1
python tools/exp/dump.py /tmp/b.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/b.npz
for i in 1 2; do
for lib in tools/exp/lib_pre.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so tools/exp/lib_pert34.so; do echo $lib; WCSVD_LIBRARY=$lib timeout 600 python tools/scenarios.py C3 "C5/2:0" 2>&1 | cut -c1-120; done
done
timeout 900 python -m pytest tests/test_gpu_l1.py tests/test_gpu_robust.py -q -x 2>&1 | tail -2
