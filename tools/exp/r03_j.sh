WCSVD_LIBRARY=tools/exp/lib_head.so python tools/exp/dump.py /tmp/a.npz | tail -1
python tools/exp/dump.py /tmp/b.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/b.npz
python -c "
import sys; sys.path.insert(0,'.')
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc; L=wc.lib(); print('occ tp64', L.wcsvd_debug_l0tp_occupancy(8,0,64), L.wcsvd_debug_l0tp_occupancy(8,1,64), 'tp32', L.wcsvd_debug_l0tp_occupancy(7,0,128))"
for i in 1 2; do
for lib in tools/exp/lib_head.so tools/exp/lib_tp4.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so tools/exp/lib_tp6.so; do echo $lib; WCSVD_LIBRARY=$lib timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-100; done
done
timeout 900 python -m pytest tests/test_gpu_l0.py tests/test_gpu_fp32.py tests/test_gpu_modes.py tests/test_gpu_host.py tests/test_gpu_robust.py -x -q 2>&1 | tail -3
