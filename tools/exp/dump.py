"""Dump S,U,V of a fixed mixed set to an .npz (for bitwise A/B comparisons of library builds)."""
import sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
out = sys.argv[1]
shapes = [(256, 256)] * 6 + [(1024, 128)] * 2 + [(300, 170), (170, 300), (600, 600), (97, 97), (1024, 1024), (64, 64), (40, 24)]
mats = [workloads.gaussian(workloads.matrix_rng(900, i), m, n) for i, (m, n) in enumerate(shapes)]
S, U, V, info = wc.svd_batched([torch.from_numpy(a).cuda() for a in mats], return_info=True)
torch.cuda.synchronize()
d = {}
for i in range(len(mats)):
    d[f"S{i}"] = S[i].cpu().numpy(); d[f"U{i}"] = U[i].cpu().numpy(); d[f"V{i}"] = V[i].cpu().numpy()
d["info"] = info.cpu().numpy()
np.savez(out, **d)
print("dumped", out, d["info"])
