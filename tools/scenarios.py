"""Device timing of svd_batched on named scenarios (development probe; bench.py is the contract).

  python tools/scenarios.py SCEN [SCEN ...] [--reps 3] [--json out.json] [--opts '{"force_w":16}']

Scenarios: a config name (C1..C5), "C5/G:r" (rank r's LPT share of C5 at G GPUs), "U:m:n:B" (B
uniform Gaussian m x n matrices, seed 900), "C3:B" / "C4:B" (first B matrices of a config).
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("WCSVD_PKG_DIR"):  # A/B experiments: import the binding + library from another tree
    sys.path.insert(0, os.environ["WCSVD_PKG_DIR"])
import workloads  # noqa: E402
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc  # noqa: E402
from paper_conf_sc_xiaopxsmmlzt22_b200 import dist as wdist  # noqa: E402


def scenario(name):
    if name.startswith("U:"):
        _, m, n, B = name.split(":")
        cfg = workloads.custom_config(name, 900, [(int(m), int(n))] * int(B))
        return cfg.sizes, cfg.make, list(range(int(B)))
    if "/" in name:
        base, rest = name.split("/")
        G, r = (int(x) for x in rest.split(":"))
        cfg = workloads.get_config(base)
        idx = wdist.lpt_partition(cfg.sizes, G)[r]
        return [cfg.sizes[k] for k in idx], cfg.make, idx
    if ":" in name:
        base, B = name.split(":")
        cfg = workloads.get_config(base, int(B))
    else:
        cfg = workloads.get_config(name)
    return cfg.sizes, cfg.make, list(range(cfg.batch))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("scen", nargs="+")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--json", default=None)
    ap.add_argument("--opts", default="{}")
    a = ap.parse_args()
    kw = {k: v for k, v in json.loads(a.opts).items() if not k.startswith("_")}
    res = []
    for s in a.scen:
        sizes, make, idx = scenario(s)
        mats = [make(k) for k in idx]
        if len(set(sizes)) == 1:
            A = torch.from_numpy(np.stack(mats)).cuda()
        else:
            A = [torch.from_numpy(x).cuda() for x in mats]
        del mats
        best = None
        for it in range(a.reps + 1):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            out = wc.svd_batched(A, return_info=True, **kw)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            if it > 0:
                best = ms if best is None else min(best, ms)
        info = out[3].cpu().numpy()
        ftb = sum(workloads.f_tb(m, n) * s_ for (m, n), s_ in zip(sizes, info))
        r = {"scenario": s, "batch": len(sizes), "ms": best, "mats_per_s": len(sizes) / best * 1e3,
             "sweeps_mean": float(info.mean()), "sweeps_max": int(info.max()), "tb_tflops": ftb / best / 1e9,
             "opts": kw}
        print(json.dumps(r), flush=True)
        res.append(r)
        del A, out
        torch.cuda.empty_cache()
    if a.json:
        os.makedirs(os.path.dirname(a.json) or ".", exist_ok=True)
        json.dump(res, open(a.json, "w"), indent=1)


if __name__ == "__main__":
    main()
