import sys; sys.path.insert(0, '.')
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
L = wc.lib()
for v, m in ((7, 32), (7, 128), (8, 64)):
    print("variant", v, "maxM", m, "fp64 occ", L.wcsvd_debug_l0tp_occupancy(v, 0, m), "fp32 occ", L.wcsvd_debug_l0tp_occupancy(v, 1, m))
