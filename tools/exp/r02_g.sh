timeout 600 python -m pytest tests/test_gpu_da.py tests/test_gpu_cluster.py -x -q 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_sanitizers.py -x -q 2>&1 | tail -3
cat > /tmp/e2e.py <<'PY'
import sys, time, torch, numpy as np
sys.path.insert(0,'.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
cfg=workloads.get_config("C5")
A=[torch.from_numpy(cfg.make(k)).pin_memory() for k in range(cfg.batch)]
ks=[min(s) for s in cfg.sizes]
out=([torch.empty(k,dtype=torch.float64).pin_memory() for k in ks],[torch.empty(k,m,dtype=torch.float64).pin_memory() for k,(m,_) in zip(ks,cfg.sizes)],[torch.empty(k,n,dtype=torch.float64).pin_memory() for k,(_,n) in zip(ks,cfg.sizes)])
for it in range(3):
    torch.cuda.synchronize(); t=time.time(); wc.svd_batched_host(A,out=out); torch.cuda.synchronize(); print(sys.argv[1], "e2e", 3000/(time.time()-t), flush=True)
PY
for t in 1 0; do WCSVD_TAILOR=$t timeout 600 python /tmp/e2e.py tailor$t; done
WCSVD_HOST_CHUNKS=1 timeout 600 python /tmp/e2e.py chunks1
