"""SURVEY §8(f2) ablations on B200 (Table I / Table V / Fig 1 analogues of the paper, PAPER.md:211-226,
408-419): for each config, time the batched SVD with the planner's choice and with one knob forced --
the EVD block width w (Table I), the path (Level 0 vs Gram vs W-cycle recursion, Alg 2), the inner
EVD sweep cap and warps per column-block pair (lanes-per-pair). Reports ms, matrices/s,
mean outer sweeps, mean inner sweeps per matrix and whether the results stay within the oracle-free
invariants (residual / orthogonality) on a few matrices. Prints one JSON object.

Usage: python tools/ablation.py [--batch B] [configs...]   (default C2 C3 C4, B = 592 = 4 waves)
"""
import argparse
import json
import sys
import os

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads  # noqa: E402
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc  # noqa: E402

KNOBS = {
    "planner": {},
    "w=8": {"force_path": wc.PATH_GRAM, "force_w": 8},
    "w=16": {"force_path": wc.PATH_GRAM, "force_w": 16},
    "wcycle(w1=64,w2=16)": {"force_path": wc.PATH_WCYCLE, "force_w": 16},
    "inner_sweeps=2": {"inner_sweeps": 2},
    "pair_warps=2": {"pair_warps": 2},
}


def run(A, kw, reps=3):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    best = None
    for _ in range(reps):
        torch.cuda.synchronize()
        ev[0].record()
        S, U, V, info = wc.svd_batched(A, return_info=True, **kw)
        ev[1].record()
        torch.cuda.synchronize()
        ms = ev[0].elapsed_time(ev[1])
        best = ms if best is None else min(best, ms)
    return best, S, U, V, info


def invariants(A, S, U, V, idx):
    worst_r, worst_o = 0.0, 0.0
    for k in idx:
        a = A[k].double().cpu().numpy()
        s, u, v = S[k].cpu().numpy(), U[k].cpu().numpy(), V[k].cpu().numpy()
        worst_r = max(worst_r, np.linalg.norm(a - (u * s) @ v.T) / np.linalg.norm(a))
        worst_o = max(worst_o, np.abs(u.T @ u - np.eye(u.shape[1])).max(), np.abs(v.T @ v - np.eye(v.shape[1])).max())
    return worst_r, worst_o


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=592)
    ap.add_argument("configs", nargs="*", default=["C2", "C3", "C4"])
    args = ap.parse_args()
    out = {"gpu": torch.cuda.get_device_name(0), "batch": args.batch, "results": {}}
    for name in args.configs:
        cfg = workloads.get_config(name, args.batch)
        A = torch.from_numpy(np.stack(cfg.matrices())).cuda()
        m, n = cfg.sizes[0]
        res = {}
        for knob, kw in KNOBS.items():
            if name == "C2" and knob in ("inner_sweeps=2", "pair_warps=2"):
                continue  # Level 0 has no inner EVD / pair executor
            try:
                p = wc.plan(m, n, force_path=kw.get("force_path", 0), force_w=kw.get("force_w", 0))
                ms, S, U, V, info = run(A, kw)
                info = info.cpu().numpy()
                r, o = invariants(A, S, U, V, range(0, args.batch, max(1, args.batch // 4)))
                res[knob] = {"ms": round(ms, 3), "matrices_per_s": round(args.batch / ms * 1e3, 1),
                             "path": p["path"], "w": p["w"], "w2": p["w2"],
                             "sweeps_mean": round(float(info.mean()), 2), "converged": bool((info > 0).all()),
                             "residual_max": float(r), "orth_max": float(o)}
            except Exception as e:  # a knob the shape does not support
                res[knob] = {"error": str(e)[:120]}
            print(name, knob, res[knob], file=sys.stderr, flush=True)
        out["results"][name] = res
    print(json.dumps(out))


if __name__ == "__main__":
    main()
