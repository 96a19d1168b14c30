"""Quick device timing of svd_batched on a config (development probe; bench.py is the contract)."""
import sys, time, json
import numpy as np, torch
sys.path.insert(0, ".")
import os
if os.environ.get("WCSVD_PKG_DIR"): sys.path.insert(0, os.environ["WCSVD_PKG_DIR"])
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
batch = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2] else None
kw = json.loads(sys.argv[3]) if len(sys.argv) > 3 else {}
cfg = workloads.get_config(name, batch)
t0 = time.time()
mats = cfg.matrices()
print("gen", time.time() - t0, flush=True)
uniform = len(set(cfg.sizes)) == 1
if uniform:
    A = torch.from_numpy(np.stack(mats)).cuda()
else:
    A = [torch.from_numpy(a).cuda() for a in mats]
for it in range(4):
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    out = wc.svd_batched(A, return_info=True, **kw)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    info = out[3].cpu().numpy()
    ftb = sum(workloads.f_tb(m, n) * s for (m, n), s in zip(cfg.sizes, info))
    print(f"{name} B={cfg.batch} ms={ms:.3f} mats/s={cfg.batch/ms*1e3:.1f} sweeps mean={info.mean():.2f} min={info.min()} max={info.max()} tbGF/s={ftb/ms/1e6:.1f}", flush=True)
