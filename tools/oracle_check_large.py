"""Parity of the largest sizes against the long-double oracle itself (too slow for the -m gpu suite:
a 1024 x 1024 oracle run takes minutes on one core). Runs the CUDA path on C5's 1024^2 matrices
k = 0, 100 (and a 1024 x 1024 with prescribed spectrum, kappa = 1e8), runs the oracle on the host cores
(one matrix per core, in parallel), and prints one JSON object with the comparison metrics
(oracle/compare.py bars: sigma 1e-12, residual 1e-12, orthogonality 1e-11, R-VEC vectors) and the sweep
counts. Usage: python tools/oracle_check_large.py [out.json]"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads  # noqa: E402
import oracle  # noqa: E402
from oracle import compare  # noqa: E402
from tests.gpu_helpers import gpu_svd_list  # noqa: E402

cfg = workloads.get_config("C5", batch=101)
mats = [cfg.make(0), cfg.make(100)]
names = ["C5[0] 1024x1024 N(0,1)", "C5[100] 1024x1024 N(0,1)"]
rng = workloads.matrix_rng(990, 0)
mats.append(workloads.prescribed(rng, 1024, 1024, np.geomspace(1.0, 1e-8, 1024)))
names.append("1024x1024 prescribed, kappa 1e8")
t0 = time.time()
S, U, V, info = gpu_svd_list(mats)
t_gpu = time.time() - t0
t0 = time.time()
So, Uo, Vo, info_o = oracle.svd_batch(mats)
t_or = time.time() - t0
out = {"what": "CUDA path vs the long-double oracle at the largest size", "oracle_seconds": t_or,
       "host_cores": os.cpu_count(), "cases": []}
for k, name in enumerate(names):
    p = compare.compare(mats[k], S[k], U[k], V[k], So[k], Uo[k], Vo[k])
    d = p.as_dict()
    d.update({"name": name, "ok": bool(p.ok()), "gpu_sweeps": int(info[k]), "oracle_sweeps": int(info_o[k])})
    out["cases"].append(d)
print(json.dumps(out, indent=1, default=float))
if len(sys.argv) > 1:
    json.dump(out, open(sys.argv[1], "w"), indent=1, default=float)
