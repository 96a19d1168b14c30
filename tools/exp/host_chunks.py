"""e2e of wcsvd_batched_host vs chunk count, and the raw copy times (development probe)."""
import os, sys, time, numpy as np, torch
sys.path.insert(0, '.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
cfg = workloads.get_config(name)
A_h = torch.from_numpy(np.stack(cfg.matrices())).pin_memory()
B, m, n = A_h.shape
k = min(m, n)
S_h = torch.empty(B, k, dtype=torch.float64).pin_memory()
U_h = torch.empty(B, k, m, dtype=torch.float64).pin_memory()
V_h = torch.empty(B, k, n, dtype=torch.float64).pin_memory()
A_d = A_h.cuda(); U_d = U_h.cuda(); V_d = V_h.cuda()
def t(f, r=3):
    best = 1e9
    for _ in range(r):
        torch.cuda.synchronize(); t0 = time.perf_counter(); f(); torch.cuda.synchronize(); best = min(best, time.perf_counter() - t0)
    return best * 1e3
print(name, "H2D A ms", round(t(lambda: A_d.copy_(A_h, non_blocking=True)), 2),
      "D2H U+V ms", round(t(lambda: (U_h.copy_(U_d, non_blocking=True), V_h.copy_(V_d, non_blocking=True))), 2))
print("device call ms", round(t(lambda: wc.svd_batched(A_d)), 2))
for c in [int(x) for x in (sys.argv[2].split(',') if len(sys.argv) > 2 else '1,2,3,4,6,8,12'.split(','))]:
    os.environ["WCSVD_HOST_CHUNKS"] = str(c)
    print("chunks", c, "e2e ms", round(t(lambda: wc.svd_batched_host(A_h, out=(S_h, U_h, V_h))), 2), flush=True)
