#!/usr/bin/env python
"""Benchmark of the batched fp64 one-sided Jacobi SVD hot path (BASELINE.json metric:
"fp64 SVD matrices/sec (S,U,V) at 1/2/4/8 B200; % of FP64 peak").

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl ours|reference]

A "step" is one call of the library over the whole batch of one BASELINE config: plan -> stage-in ->
every sweep of Gram / EVD / update / off-test (or the Level-0 kernel) -> finalisation, producing S, U
and V for every matrix. The default workload is C5 (3,000 mixed-size matrices, m, n in [32, 1024],
30 x 1024^2): the largest config, one of the 1/2/4/8-GPU configs, and the one that exercises the
planner, Level 0 and the Gram path together. --config C1..C4 selects another.

Multi-GPU (north_star): the FIXED config batch is partitioned over the N ranks by the
greedy LPT split of dist.lpt_partition (estimated cost F_tb, largest first); every rank regenerates
only its own matrices from (seed, k), factors them with no collective on the data path, and the
device time is the max over ranks (strong scaling). The end-to-end leg (`e2e`) is the public host-
buffer call (wcsvd_batched_host: H2D, kernels, D2H inside) on every rank followed by the one NCCL
gather of S to rank 0 (dist.gather_sigma), all inside the timed region. `--gpus N` without a
torchrun environment re-launches itself under torch.distributed.run with N ranks.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads  # noqa: E402

METRIC = "fp64 SVD matrices/sec (S,U,V)"
FP64_PEAK_NOMINAL_TFLOPS = 148 * 64 * 2 * 1.965e9 / 1e12  # 37.2: SMs x FP64 FMA/clk x 2 x max clock


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5", choices=list(workloads.CONFIGS))
    ap.add_argument("--batch", type=int, default=None, help="truncate the config to its first B matrices")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    return ap.parse_args()


# ------------------------------------------------------------------------------------------------
# clocks sampled during the timed region (NVML)
class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons)}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons - {"gpu_idle"}), "samples": len(self.samples)}


def host_cpu():
    model = None
    try:
        for line in subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout.splitlines():
            if line.startswith("Model name"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"model": model, "nproc": os.cpu_count()}


# ------------------------------------------------------------------------------------------------
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def relaunch(args) -> int:
    """--gpus N outside torchrun: re-run this script under torch.distributed.run with N ranks."""
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def workload(args):
    """(config, sizes of the fixed batch, make(k))."""
    cfg = workloads.get_config(args.config, args.batch)
    return cfg, list(cfg.sizes), cfg.make


def cpu_baseline(sizes, make, idx_pool, seconds_target):
    """The oracle (T = double instantiation, OpenMP over matrices) on a bounded, evenly strided
    sample of the workload, on the host cores (rank 0, N = 1 only)."""
    import oracle

    lib = oracle.build()
    try:  # a -march=native copy for this host (scratch path; the portable build is the fallback)
        lib = oracle.build(native=True, out="/tmp/liboracle_native_%d.so" % os.getpid(), force=True)
    except Exception:
        pass
    cores = os.cpu_count() or 1
    # calibrate on an evenly strided handful, then size the sample for ~seconds_target
    n_cal = min(len(idx_pool), max(cores, 8))
    cal = idx_pool[::max(1, len(idx_pool) // n_cal)][:n_cal]
    t0 = time.perf_counter()
    oracle.svd_batch([make(k) for k in cal], precision="d", threads=cores, lib_path=lib)
    per_cost = (time.perf_counter() - t0) / sum(workloads.f_tb(*sizes[k]) for k in cal)
    tot_cost = sum(workloads.f_tb(*sizes[k]) for k in idx_pool)
    frac = min(1.0, seconds_target / max(per_cost * tot_cost, 1e-9))
    step = max(1, int(round(1.0 / frac)))
    sel = idx_pool[::step]
    mats = [make(k) for k in sel]
    t0 = time.perf_counter()
    _, _, _, info = oracle.svd_batch(mats, precision="d", threads=cores, lib_path=lib)
    dt = time.perf_counter() - t0
    # matrices/s of the whole workload at the sample's cost rate (mixed sizes: scaled by F_tb share)
    sel_cost = sum(workloads.f_tb(*sizes[k]) for k in sel)
    value = len(idx_pool) / (dt * tot_cost / sel_cost)
    cores = oracle.threads_in_effect(lib)
    return {"value": value, "unit": "matrices/s", "cores": cores, "kind": "oracle",
            "sample": f"every {step}th matrix of the workload ({len(sel)} of {len(idx_pool)}), cyclic one-sided "
                      f"Jacobi, oracle/oracle.c T=double, OpenMP x{cores}, {dt:.1f} s; whole-workload rate "
                      f"extrapolated by the sample's F_tb share ({sel_cost / tot_cost:.4f})",
            "sample_indices": [int(k) for k in sel[:64]], "oracle_sweeps_mean": float(np.mean(info)),
            "host_cpu": host_cpu()}, sel, info


def run_reference(args, world, rank):
    """--impl reference: the CPU oracle as the reference arm (no installable reference exists).
    Rank 0 alone runs it; other ranks exit without work."""
    if rank != 0:
        return
    import oracle

    cfg, sizes, make = workload(args)
    lib = oracle.build()
    cores = os.cpu_count() or 1
    idx = list(range(len(sizes)))
    cal = idx[::max(1, len(idx) // max(cores, 8))][:max(cores, 8)]
    t0 = time.perf_counter()
    oracle.svd_batch([make(k) for k in cal], precision="d", threads=cores, lib_path=lib)
    per_cost = (time.perf_counter() - t0) / sum(workloads.f_tb(*sizes[k]) for k in cal)
    tot_cost = sum(workloads.f_tb(*sizes[k]) for k in idx)
    budget = 150.0 / max(args.warmup + args.steps, 1)  # whole run within a few minutes
    step = max(1, int(round(per_cost * tot_cost / budget)))
    sel = idx[::step]
    sel_cost = sum(workloads.f_tb(*sizes[k]) for k in sel)
    mats = [make(k) for k in sel]
    times = []
    for s in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.svd_batch(mats, precision="d", threads=cores, lib_path=lib)
        if s >= args.warmup:
            times.append(time.perf_counter() - t0)
    t_sample = sum(times) / len(times)
    t_whole = t_sample * tot_cost / sel_cost  # extrapolated by F_tb share
    value = len(idx) / t_whole
    cores = oracle.threads_in_effect(lib)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "matrices/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_whole,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": f"{args.config}: {cfg.description}", "batch": len(idx),
                                            "per_step_sample": len(sel), "sample_stride": step},
            "cpu_baseline": {"value": value, "unit": "matrices/s", "cores": cores, "kind": "oracle",
                             "sample": f"every {step}th matrix ({len(sel)} of {len(idx)}) per step, oracle "
                                       f"T=double, OpenMP x{cores}, {t_sample:.1f} s per step; whole-workload "
                                       f"rate extrapolated by F_tb share {sel_cost / tot_cost:.4f}",
                             "host_cpu": host_cpu()},
            "e2e": {"value": value, "unit": "matrices/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    world, rank, local = dist_env()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch(args))
    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    import torch
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
    from paper_conf_sc_xiaopxsmmlzt22_b200 import dist as wdist

    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (the library has no CPU fallback)")
    ndev = torch.cuda.device_count()
    local_dev = local % ndev  # == local on a real box (one process per GPU)
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    tdist = None
    if world > 1:
        import torch.distributed as tdist
        if ndev >= world:
            tdist.init_process_group("nccl", device_id=dev)
        else:  # ranks sharing a GPU (1-GPU development box): NCCL refuses duplicate devices
            tdist.init_process_group("gloo")

    cfg, sizes_all, make = workload(args)
    B_total = len(sizes_all)
    parts = wdist.lpt_partition(sizes_all, world)
    mine = parts[rank]
    sizes = [sizes_all[k] for k in mine]
    B = len(sizes)
    uniform = len(set(sizes)) == 1
    t0 = time.time()
    host = [np.ascontiguousarray(make(k)) for k in mine]
    gen_s = time.time() - t0

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev if tdist.get_backend() == "nccl" else "cpu")
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev if tdist.get_backend() == "nccl" else "cpu")
        tdist.all_reduce(t, op=tdist.ReduceOp.SUM)
        return float(t.item())

    def barrier():
        if world > 1:
            tdist.barrier()
        torch.cuda.synchronize()

    # device-resident inputs and preallocated outputs
    if uniform:
        m, n = sizes[0]
        k = min(m, n)
        A_h = torch.from_numpy(np.stack(host)).pin_memory()
        A = A_h.to(dev)
        out = (torch.empty(B, k, device=dev, dtype=torch.float64), torch.empty(B, k, m, device=dev, dtype=torch.float64),
               torch.empty(B, k, n, device=dev, dtype=torch.float64))
        call = lambda X: wc.svd_batched(X, out=out, return_info=True)
    else:
        A_h = [torch.from_numpy(a).pin_memory() for a in host]
        A = [a.to(dev) for a in A_h]
        call = lambda X: wc.svd_batched(X, return_info=True)
    in_bytes = sum(mm * nn for (mm, nn) in sizes) * 8
    out_bytes = sum(min(mm, nn) * (1 + mm + nn) for (mm, nn) in sizes) * 8
    del host
    stream = torch.cuda.current_stream()

    # warm-up (also yields sweeps per matrix for the algorithmic flop count)
    for _ in range(args.warmup):
        res = call(A)
    torch.cuda.synchronize()
    info = res[3].cpu().numpy()
    flops_alg = float(sum(workloads.f_tb(mm, nn) * max(int(s), 0) for (mm, nn), s in zip(sizes, info)))

    # ---- timed region: device-resident inputs, K steps, CUDA events on the launching stream ----
    barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local_dev) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            res = call(A)
        ev1.record(stream)
        barrier()
    ms = max_over_ranks(ev0.elapsed_time(ev1))
    ms_step = ms / args.steps
    value = B_total * args.steps / (ms * 1e-3)
    flops_all = sum_over_ranks(flops_alg)

    # ---- dominant kernel (roofline): the Gram-path bucket with the most work (or the Level-0 bucket),
    # timed on its own as one launch on this stream (+ the completion pass), same events ----
    plans = [wc.plan(mm, nn) for (mm, nn) in sizes]
    keyw = {}
    for (mm, nn), p, s in zip(sizes, plans, info):
        key = (p["path"], p["variant"])
        keyw[key] = keyw.get(key, 0.0) + workloads.f_tb(mm, nn) * max(int(s), 0)
    dom_key = max(keyw, key=keyw.get)
    dom_idx = [i for i, p in enumerate(plans) if (p["path"], p["variant"]) == dom_key]
    names = {wc.PATH_L0: "l0_jacobi_kernel", wc.PATH_GRAM: "l1_gram_kernel", wc.PATH_WCYCLE: "l1_gram_kernel"}
    dom_name = names[dom_key[0]]
    if dom_key[0] == wc.PATH_L0 and dom_key[1] in wc.L0_TWO_PHASE_VARIANTS:
        dom_name = "l0tp_kernel"
    if len(dom_idx) == B:
        k_ms, k_flops = ms_step, flops_alg
    else:
        sub = [A[i] for i in dom_idx]
        for _ in range(2):
            wc.svd_batched(sub, return_info=True)
        torch.cuda.synchronize()
        k0 = torch.cuda.Event(enable_timing=True)
        k1 = torch.cuda.Event(enable_timing=True)
        k0.record(stream)
        for _ in range(args.steps):
            wc.svd_batched(sub, return_info=True)
        k1.record(stream)
        torch.cuda.synchronize()
        k_ms = k0.elapsed_time(k1) / args.steps
        k_flops = sum(workloads.f_tb(*sizes[i]) * max(int(info[i]), 0) for i in dom_idx)
    achieved_tf = k_flops / (k_ms * 1e-3) / 1e12
    peaks = {}
    pj = os.path.join(ROOT, "profiles", "peaks_fp64_r01.json")
    if os.path.exists(pj):
        try:
            peaks = json.load(open(pj))
        except Exception:
            peaks = {}
    # FP64 pipe peak for the kernel's own instruction kind: DMMA.8x8x4 (Gram path) or DFMA (Level 0)
    pkey = "fp64_dfma_tflops" if dom_key[0] == wc.PATH_L0 else "fp64_dmma_tflops"
    peak = float(peaks.get(pkey, 0) or 0) or FP64_PEAK_NOMINAL_TFLOPS
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_summary_r02.json")
    if os.path.exists(prof):  # ncu --set full dram bytes of the same kernel (profiles/), per matrix x matrices
        try:
            per = json.load(open(prof)).get(args.config, {}).get("dram_bytes_per_matrix")
            traffic = None if per is None else per * len(dom_idx)
        except Exception:
            traffic = None
    roofline = {"bound": "alu" if dom_key[0] == wc.PATH_L0 else "tensor", "achieved": achieved_tf, "peak": peak,
                "unit": "TFLOP/s", "frac": achieved_tf / peak, "traffic": traffic, "kernel": dom_name,
                "launch": f"plan bucket path={dom_key[0]} variant={dom_key[1]}: {len(dom_idx)} of this rank's {B} "
                          f"matrices, one launch on the bench stream (+ completion pass), {k_ms:.2f} ms",
                "algorithmic_flops_per_launch": k_flops,
                "peak_note": (f"measured FP64 peak ({pkey}), profiles/peaks_fp64_r01.json (MEASURED_PEAKS.json has "
                              "no fp64 entry; nominal 37.2 = 148 SM x 64 FMA/clk x 2 x 1.965 GHz)")
                if peaks else "nominal FP64 37.2 TF/s (no measured fp64 peak found)",
                "flops": "textbook F_tb(M,N)=N(N-1)/2(8M+6N) x GPU sweeps used, summed over the launch's matrices"}

    # ---- e2e: the public end-to-end call with HOST buffers (wcsvd_batched_host: pinned inputs -> H2D ->
    # kernels -> D2H of S, U, V inside the library), then the one gather of S to rank 0 (NCCL) ----
    if uniform:
        k_ = min(sizes[0])
        S_h = torch.empty(B, k_, dtype=torch.float64).pin_memory()
        U_h = torch.empty(B, k_, sizes[0][0], dtype=torch.float64).pin_memory()
        V_h = torch.empty(B, k_, sizes[0][1], dtype=torch.float64).pin_memory()
        out_h = (S_h, U_h, V_h)
    else:
        ks_ = [min(mm, nn) for (mm, nn) in sizes]
        out_h = ([torch.empty(k, dtype=torch.float64).pin_memory() for k in ks_],
                 [torch.empty(k, mm, dtype=torch.float64).pin_memory() for k, (mm, _) in zip(ks_, sizes)],
                 [torch.empty(k, nn, dtype=torch.float64).pin_memory() for k, (_, nn) in zip(ks_, sizes)])

    def e2e_step():
        S_res = wc.svd_batched_host(A_h, out=out_h)[0]
        if world > 1:
            S_list = list(S_res) if uniform else S_res
            wdist.gather_sigma(mine, S_list, sizes_all)

    e2e_step()
    barrier()
    ee0 = torch.cuda.Event(enable_timing=True)
    ee1 = torch.cuda.Event(enable_timing=True)
    e_steps = max(1, min(args.steps, 3))
    ee0.record(stream)
    for _ in range(e_steps):
        e2e_step()
    ee1.record(stream)
    barrier()
    e_ms = max_over_ranks(ee0.elapsed_time(ee1))
    e2e_value = B_total * e_steps / (e_ms * 1e-3)
    h2d_all = sum_over_ranks(in_bytes)
    d2h_all = sum_over_ranks(out_bytes)
    launches = sum_over_ranks(len({(p["path"], p["variant"]) for p in plans}) + 1)

    line = {"metric": METRIC, "value": value, "unit": "matrices/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.config}: {cfg.description}", "batch": B_total,
                       "sizes": f"{sizes[0][0]}x{sizes[0][1]}" if len(set(sizes_all)) == 1 else "mixed",
                       "parallelism": f"batch-parallel x{world}: LPT split of the fixed batch by F_tb "
                                      f"(rank 0 holds {B} matrices), no collective on the data path",
                       "l2": f"inputs larger than L2 ({in_bytes / 1e6:.0f} MB on rank 0 vs 126 MB); no flush"
                       if in_bytes > 126e6 else f"inputs {in_bytes / 1e6:.1f} MB fit L2; no flush",
                       "gen_seconds": round(gen_s, 2)},
            "sweeps": {"gpu_mean": float(np.mean(info)), "gpu_min": int(info.min()), "gpu_max": int(info.max())},
            "sweep_normalised_tflops": flops_all / (ms_step * 1e-3) / 1e12,
            "e2e": {"value": e2e_value, "unit": "matrices/s", "h2d_bytes_per_step": int(h2d_all),
                    "d2h_bytes_per_step": int(d2h_all),
                    "what": "wcsvd_batched_host on every rank (pinned host A in, S, U, V out: staged H2D / kernels / D2H pipeline, or for compute-heavy batches such as C5 the zero-copy route where the kernels read A and write S, U, V in the mapped host buffers; DESIGN.md 5.6)"
                            + (" + one NCCL all_gather of S to rank 0 (dist.gather_sigma)" if world > 1 else "")},
            "gpu_launches": int(launches) * args.steps,
            "clocks": clk.summary(),
            "roofline": roofline}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cb, sel, oinfo = cpu_baseline(sizes_all, make, list(range(B_total)), args.cpu_seconds)
        pos = {k: i for i, k in enumerate(mine)}
        line["cpu_baseline"] = cb
        line["sweeps"]["oracle_mean_on_sample"] = float(np.mean(oinfo))
        line["sweeps"]["gpu_mean_on_sample"] = float(np.mean([info[pos[k]] for k in sel]))
    if world > 1:
        tdist.barrier()
        tdist.destroy_process_group()
    if rank == 0:
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
