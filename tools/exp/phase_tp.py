"""Run a config with the phase-profiling build and print the two-phase Level-0 cycle split."""
import ctypes, sys, json
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
name, batch = sys.argv[1], int(sys.argv[2])
kw = json.loads(sys.argv[3]) if len(sys.argv) > 3 else {}
cfg = workloads.get_config(name, batch)
A = torch.from_numpy(np.stack(cfg.matrices())).cuda()
L = wc.lib()
buf = (ctypes.c_ulonglong * 8)()
wc.svd_batched(A, **kw); torch.cuda.synchronize()
L.wcsvd_debug_tp_cycles(buf, 1)
wc.svd_batched(A, **kw); torch.cuda.synchronize()
L.wcsvd_debug_tp_cycles(buf, 0)
nw = buf[5]  # warp-steps are counted per warp (lane 0 of each warp adds)
steps = buf[5]
print("per warp-step cycles: phase1+bar1 %.0f  serial+bar2 %.0f  rotate %.0f" % (buf[0] / steps, buf[1] / steps, buf[2] / steps))
if buf[6]:
    print("per warp V-sweep cycles: V %.0f  park/unpark %.0f  (V sweeps %d)" % (buf[3] / buf[6], buf[4] / buf[6], buf[6]))
tot = buf[0] + buf[1] + buf[2] + buf[3] + buf[4]
for i, n in enumerate(["phase1+bar1", "serial+bar2", "rotate", "V", "park"]):
    print(f"{n:12s} {100 * buf[i] / tot:5.1f}%")
