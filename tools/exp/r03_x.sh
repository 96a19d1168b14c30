WCSVD_LIBRARY=tools/exp/lib_pre.so python tools/exp/dump.py /tmp/a.npz | tail -1
python tools/exp/dump.py /tmp/b.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/b.npz
for i in 1 2; do
WCSVD_LIBRARY=tools/exp/lib_pre.so timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-100
timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-100
done
