"""Plan search on B200 (the paper's auto-tuning engine, Tables II-III,
V): for a grid of matrix shapes, time every path / EVD width the library can run -- Level 0 (when the
matrix fits one CTA), the flat Gram path with w = 8 or 16, the W-cycle (w1 = 64 super-blocks over
w2 = 8 or 16 sub-blocks), the group (i) PANEL path (w = 16) -- on a batch that fills the GPU (tailoring off: one CTA per matrix), and
record the per-matrix time and the outer sweeps. tools/gen_plan_table.py turns the result into the
planner's table (csrc/plan_table.h). Prints / writes one JSON object.

Usage: python tools/autotune.py [--out profiles/autotune_r02.json] [--quick]
"""
import argparse
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc  # noqa: E402

CANDS = {
    "L0": {"force_path": wc.PATH_L0},
    "gram_w8": {"force_path": wc.PATH_GRAM, "force_w": 8},
    "gram_w16": {"force_path": wc.PATH_GRAM, "force_w": 16},
    "wcycle_w2_16": {"force_path": wc.PATH_WCYCLE, "force_w": 16},
    "wcycle_w2_8": {"force_path": wc.PATH_WCYCLE, "force_w": 8},
    "panel_w16": {"force_path": wc.PATH_PANEL},
}


def shapes(quick=False):
    Ns = [3, 8, 16, 24, 32, 40, 48, 56, 64, 72, 80, 88, 96, 104, 128, 160, 192, 256, 352, 512, 768, 1024]
    Ns = Ns if not quick else [72, 160, 512]
    out = []
    for N in Ns:
        for r in (1.0, 1.6, 3.0, 8.0, 32.0):
            M = min(1024, int(round(N * r)))
            if (M, N) not in out:
                out.append((M, N))
    return out


def f_tb(M, N):
    return N * (N - 1) / 2.0 * (8.0 * M + 6.0 * N)


def batch_for(M, N):
    # >= one full wave of CTAs (148 SMs x up to 4 resident) and ~2e12 textbook flops (~12 sweeps)
    return int(min(4000, max(296, 2.0e12 / (12 * f_tb(M, N)))))


def time_one(A, kw, reps=2):
    reps = 1 if A.shape[1] * A.shape[2] >= 512 * 512 else reps
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    best, info = None, None
    for _ in range(reps + 1):
        torch.cuda.synchronize()
        ev[0].record()
        S, U, V, info = wc.svd_batched(A, return_info=True, cluster_ctas=1, **kw)
        ev[1].record()
        torch.cuda.synchronize()
        ms = ev[0].elapsed_time(ev[1])
        best = ms if best is None else min(best, ms)
    return best, info


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--cands", default=None, help="comma-separated subset of the candidates")
    ap.add_argument("--merge", default=None, help="add the new candidates to this earlier result")
    a = ap.parse_args()
    cands = {k: v for k, v in CANDS.items() if a.cands is None or k in a.cands.split(",")}
    prev = {}
    if a.merge:
        for r in json.load(open(a.merge))["shapes"]:
            prev[(r["m"], r["n"])] = r
    g = torch.Generator(device="cuda").manual_seed(2602)
    res = []
    t0 = time.time()
    for (M, N) in shapes(a.quick):
        B = batch_for(M, N)
        row = prev.get((M, N)) or {"m": M, "n": N, "batch": B, "planner": wc.plan(M, N), "ms_per_matrix": {},
                                   "sweeps": {}}
        B = row["batch"]
        A = torch.randn(B, M, N, dtype=torch.float64, device="cuda", generator=g)
        for name, kw in cands.items():
            try:
                wc.plan(M, N, kw.get("force_path", 0), kw.get("force_w", 0))
            except wc.WcsvdError:
                continue
            ms, info = time_one(A, kw)
            if int((info <= 0).sum()) > 0:
                row.setdefault("not_converged", {})[name] = int((info <= 0).sum())
            row["ms_per_matrix"][name] = ms / B
            row["sweeps"][name] = float(info.float().mean())
        best = min(row["ms_per_matrix"], key=row["ms_per_matrix"].get)
        row["best"] = best
        print(json.dumps({k: row[k] for k in ("m", "n", "batch", "best", "ms_per_matrix", "sweeps")}), flush=True)
        res.append(row)
        del A
        torch.cuda.empty_cache()
    out = {"gpu": torch.cuda.get_device_name(0), "seconds": time.time() - t0, "shapes": res,
           "how": "randn fp64 batches on the device, device time of svd_batched (best of 2 after a warm-up), "
                  "cluster_ctas = 1 (throughput per matrix, no tailoring)"}
    if a.out:
        os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
        json.dump(out, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
