cat > /tmp/c1time.py <<'PY'
import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
cfg = workloads.get_config("C1")
A = torch.from_numpy(np.stack(cfg.matrices())).cuda()
S = torch.empty(100, 32, dtype=torch.float64, device='cuda'); U = torch.empty(100, 32, 32, dtype=torch.float64, device='cuda'); V = torch.empty_like(U)
for i in range(5): wc.svd_batched(A, out=(S, U, V))
torch.cuda.synchronize()
for i in range(4):
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); t = time.perf_counter(); e0.record()
    wc.svd_batched(A, out=(S, U, V))
    t1 = time.perf_counter(); e1.record(); torch.cuda.synchronize(); t2 = time.perf_counter()
    print("host call %.3f ms, event %.3f ms, wall %.3f ms" % ((t1 - t) * 1e3, e0.elapsed_time(e1), (t2 - t) * 1e3))
PY
for lib in tools/exp/lib_head.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so; do echo $lib; WCSVD_LIBRARY=$lib python /tmp/c1time.py; WCSVD_LIBRARY=$lib ncu --metrics gpu__time_duration.sum --clock-control none --csv python /tmp/c1time.py 2>/dev/null | grep -E "l0_|complete" | awk -F'","' '{print $5, $(NF)}' | tail -4; done
