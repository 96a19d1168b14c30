"""Small mixed batch for compute-sanitizer runs (L0 variants, L1 flat w=8/16, W-cycle)."""
import sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
mode = sys.argv[1] if len(sys.argv) > 1 else "mixed"
shapes = [(32, 32), (64, 64), (40, 24), (24, 40), (130, 100), (100, 150), (256, 160), (17, 9)]
mats = [workloads.gaussian(workloads.matrix_rng(777, i), m, n) for i, (m, n) in enumerate(shapes)]
kw = {}
if mode == "wcycle":
    mats = [mats[4], mats[6]]
    kw = dict(force_path=wc.PATH_WCYCLE)
S, U, V, info = wc.svd_batched([torch.from_numpy(a).cuda() for a in mats], return_info=True, **kw)
torch.cuda.synchronize()
print("info", info.cpu().numpy())
