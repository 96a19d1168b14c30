"""Run a config with the phase-profiling build and print the Level-1 cycle split."""
import ctypes, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
name, batch = sys.argv[1], int(sys.argv[2])
cfg = workloads.get_config(name, batch)
A = torch.from_numpy(np.stack(cfg.matrices())).cuda()
L = wc.lib()
buf = (ctypes.c_ulonglong * 12)()
wc.svd_batched(A); torch.cuda.synchronize()
L.wcsvd_debug_phase_cycles(buf, 1)
wc.svd_batched(A); torch.cuda.synchronize()
L.wcsvd_debug_phase_cycles(buf, 0)
names = ["gram", "offtest", "evd", "ns+jfrag", "apply_A", "apply_V"]
tot = sum(buf[i] for i in range(6))
for i, n in enumerate(names):
    print(f"{n:9s} {buf[i]/tot*100:5.1f}%  {buf[i]:.3e} warp-cycles")
print(f"EVD steps {buf[6]*31}, rotation-free {buf[8]} ({100*buf[8]/max(buf[6]*31,1):.1f}%)")
print(f"pairs {buf[7]}, with EVD {buf[6]}; cycles/pair {tot/max(buf[7],1):.0f}; EVD cycles/call {buf[2]/max(buf[6],1):.0f}; gram/pair {buf[0]/max(buf[7],1):.0f}; apply_A/call {buf[4]/max(buf[6],1):.0f} apply_V/call {buf[5]/max(buf[6],1):.0f}")
print(f"near-diagonal B among pairs with an EVD: <=1e-2 {buf[10]/max(buf[6],1)*100:.1f}%  <=2e-3 {buf[9]/max(buf[6],1)*100:.1f}%  <=1e-4 {buf[11]/max(buf[6],1)*100:.1f}%")
