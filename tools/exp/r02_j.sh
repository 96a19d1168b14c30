timeout 900 python -m pytest tests/test_gpu_fp32.py tests/test_gpu_l1.py tests/test_gpu_cluster.py -x -q 2>&1 | tail -5
cat > /tmp/f32t.py <<'PY'
import sys, torch, numpy as np
sys.path.insert(0,'.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
for name in ("C3","C4"):
    cfg=workloads.get_config(name)
    A=torch.from_numpy(np.stack(cfg.matrices())).cuda()
    for dt in (torch.float64, torch.float32):
        X=A.to(dt)
        for it in range(3):
            e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(); e0.record(); S,U,V,info=wc.svd_batched(X, return_info=True); e1.record(); torch.cuda.synchronize()
        print(name, dt, e0.elapsed_time(e1), "ms", cfg.batch/e0.elapsed_time(e1)*1e3, "mats/s sweeps", info.float().mean().item(), flush=True)
PY
timeout 900 python /tmp/f32t.py
