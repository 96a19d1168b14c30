WCSVD_LIBRARY=tools/exp/lib_head.so python tools/exp/dump.py /tmp/a.npz | tail -1
python tools/exp/dump.py /tmp/b.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/b.npz
WCSVD_L1_NW=4 WCSVD_L1_RES4=3 WCSVD_LIBRARY=tools/exp/lib_min3.so python tools/exp/dump.py /tmp/c.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/c.npz
for i in 1 2; do
WCSVD_LIBRARY=tools/exp/lib_head.so timeout 600 python tools/scenarios.py C3 C4 "C5/4:0" 2>&1 | cut -c1-120
timeout 600 python tools/scenarios.py C3 C4 "C5/4:0" 2>&1 | cut -c1-120
WCSVD_L1_NW=4 WCSVD_L1_RES4=3 WCSVD_LIBRARY=tools/exp/lib_min3.so timeout 600 python tools/scenarios.py C3 C4 "C5/4:0" 2>&1 | cut -c1-120
done
