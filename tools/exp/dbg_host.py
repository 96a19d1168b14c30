import sys, os, numpy as np, torch
sys.path.insert(0, '.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
cfg = workloads.get_config("C5", batch=int(sys.argv[1]) if len(sys.argv) > 1 else 40)
mats = [torch.from_numpy(a).pin_memory() for a in cfg.matrices()]
print([tuple(a.shape) for a in mats][:10], flush=True)
try:
    S, U, V, info = wc.svd_batched_host(mats, return_info=True)
    print("ok", info[:10])
except Exception as e:
    print("ERR", e)
