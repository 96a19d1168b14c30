"""Small mixed batch for compute-sanitizer runs (L0 variants, L1 flat w=8/16, W-cycle, 4-CTA clusters, the host-buffer pipeline)."""
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
if mode == "cluster":  # Gram-path matrices over 4-CTA clusters (w = 8 and 16 shapes)
    mats = [mats[4], workloads.gaussian(workloads.matrix_rng(778, 0), 120, 160), mats[6]]
    kw = dict(cluster_ctas=4)
if mode == "host":  # wcsvd_batched_host: chunked copy / compute pipeline, uniform and mixed
    A = torch.from_numpy(np.stack([workloads.gaussian(workloads.matrix_rng(779, i), 64, 64) for i in range(40)]))
    S, U, V, info = wc.svd_batched_host(A.pin_memory(), return_info=True)
    print("info", info[:8])
    S, U, V, info = wc.svd_batched_host([torch.from_numpy(a).pin_memory() for a in mats], return_info=True)
    print("info", info)
    sys.exit(0)
S, U, V, info = wc.svd_batched([torch.from_numpy(a).cuda() for a in mats], return_info=True, **kw)
torch.cuda.synchronize()
print("info", info.cpu().numpy())
