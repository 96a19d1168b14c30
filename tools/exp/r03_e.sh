timeout 300 python tools/scenarios.py C2 C1 2>&1 | cut -c1-110
WCSVD_PKG_DIR=tools/exp/old_pkg timeout 300 python tools/scenarios.py C2 C1 2>&1 | cut -c1-110
python - <<'PY'
import ctypes, time, numpy as np, torch, sys
sys.path.insert(0,'.')
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
L = wc.lib(); L.wcsvd_workspace_size.restype = ctypes.c_size_t
B=10000; m = np.full(B,64,np.int32); n=np.full(B,64,np.int32)
for i in range(3):
    t=time.time(); L.wcsvd_workspace_size(B, m.ctypes.data, n.ctypes.data); print("plan ms", (time.time()-t)*1e3)
A = torch.randn(B,64,64,dtype=torch.float64,device='cuda')
for i in range(4):
    torch.cuda.synchronize(); t=time.time(); wc.svd_batched(A); t1=time.time(); torch.cuda.synchronize(); t2=time.time()
    print("host call ms %.2f total %.2f" % ((t1-t)*1e3, (t2-t)*1e3))
PY
