#!/usr/bin/env python
"""Benchmark of the batched fp64 one-sided Jacobi SVD hot path (BASELINE.json metric:
"fp64 SVD matrices/sec (S,U,V) at 1/2/4/8 B200; % of FP64 peak").

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl ours|reference]

A "step" is one call of the library (wcsvd_batched through the Python binding) over the whole
per-GPU batch of one BASELINE config: plan -> stage-in -> every sweep of Gram/EVD/update/off-test
(or the Level-0 kernel) -> finalisation, producing S, U and V for every matrix. The default
workload is configs[1] (C2: 10,000 x 64x64); --config C1..C5 selects another (C3-C5 exercise the
Level-1 Gram path). Multi-GPU: one process per GPU (torchrun), weak scaling -- every rank factors
its own full batch of distinct seeded matrices (indices offset by rank), no collective on the data
path; time = max over ranks of the CUDA-event time. Inputs are larger than L2 for C2-C5 (stated in
config.l2). Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
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
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2", choices=list(workloads.CONFIGS))
    ap.add_argument("--batch", type=int, default=None, help="override the per-GPU batch (default: the config's)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=None)
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


# ------------------------------------------------------------------------------------------------
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def local_config(cfg_name, batch, rank):
    """This rank's batch: the config's matrices with indices offset by rank * B (weak scaling)."""
    base = workloads.get_config(cfg_name)
    B = batch or base.batch
    idx = [rank * B + k for k in range(B)]
    if cfg_name == "C5":
        sizes = [base.sizes[k % base.batch] for k in idx]
        make = lambda k: workloads.gaussian(workloads.matrix_rng(base.seed, k), *base.sizes[k % base.batch])
    else:
        sizes = [base.sizes[0]] * B
        make = base.make
    return base, idx, sizes, make


def cpu_baseline(cfg_name, sizes_idx, make, seconds_target=15.0, sample=None):
    """The oracle (T = double instantiation, OpenMP over matrices) on a bounded sample, host cores."""
    import oracle

    lib = oracle.build()
    try:  # a -march=native copy for this host (scratch path; the portable build is the fallback)
        lib = oracle.build(native=True, out="/tmp/liboracle_native_%d.so" % os.getpid(), force=True)
    except Exception:
        pass
    cores = os.cpu_count() or 1
    # calibrate on a few matrices, then size the sample for ~seconds_target
    n_cal = min(len(sizes_idx), max(cores, 8))
    mats = [make(k) for k in sizes_idx[:n_cal]]
    t0 = time.perf_counter()
    oracle.svd_batch(mats, precision="d", threads=cores, lib_path=lib)
    dt = time.perf_counter() - t0
    per = dt / n_cal
    n = sample or int(min(len(sizes_idx), max(n_cal, seconds_target / max(per, 1e-9))))
    step = max(1, len(sizes_idx) // n)
    sel = sizes_idx[::step][:n]
    mats = [make(k) for k in sel]
    t0 = time.perf_counter()
    _, _, _, info = oracle.svd_batch(mats, precision="d", threads=cores, lib_path=lib)
    dt = time.perf_counter() - t0
    cores = oracle.threads_in_effect(lib)
    return {"value": len(sel) / dt, "unit": "matrices/s", "cores": cores, "kind": "oracle",
            "sample": f"{len(sel)} of the config's matrices (every {step}th), cyclic one-sided Jacobi, "
                      f"oracle/oracle.c T=double, OpenMP x{cores}; {dt:.1f} s; mean sweeps {float(np.mean(info)):.2f}"}


def run_reference(args, world, rank):
    """--impl reference: the CPU oracle as the reference arm (no installable reference exists)."""
    if rank != 0:
        return
    base, idx, sizes, make = local_config(args.config, args.batch, 0)
    import oracle
    lib = oracle.build()
    cores = os.cpu_count() or 1
    cal = [make(k) for k in idx[:cores]]
    t0 = time.perf_counter()
    oracle.svd_batch(cal, precision="d", threads=cores, lib_path=lib)
    per = (time.perf_counter() - t0) / len(cal)
    n = int(max(cores, min(len(idx), 8.0 / max(per, 1e-9))))  # ~8 s per step
    times = []
    mats = [make(k) for k in idx[:n]]
    for s in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.svd_batch(mats, precision="d", threads=cores, lib_path=lib)
        if s >= args.warmup:
            times.append(time.perf_counter() - t0)
    value = n * len(times) / sum(times)
    cores = oracle.threads_in_effect(lib)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "matrices/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": f"{args.config}: {base.description}",
                                            "per_step_sample": n},
            "cpu_baseline": {"value": value, "unit": "matrices/s", "cores": cores, "kind": "oracle",
                             "sample": f"{n} matrices per step, oracle T=double, OpenMP x{cores}"},
            "e2e": {"value": value, "unit": "matrices/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    world, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    import torch
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc

    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (the library has no CPU fallback)")
    ndev = torch.cuda.device_count()
    local_dev = local % ndev  # == local on a real box (one process per GPU)
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    if world > 1:
        import torch.distributed as dist
        if ndev >= world:
            dist.init_process_group("nccl", device_id=dev)
        else:  # ranks sharing a GPU (1-GPU development box): NCCL refuses duplicate devices
            dist.init_process_group("gloo")

    base, idx, sizes, make = local_config(args.config, args.batch, rank)
    B = len(idx)
    uniform = len(set(sizes)) == 1
    t0 = time.time()
    host = [np.ascontiguousarray(make(k)) for k in idx]
    gen_s = time.time() - t0

    # device-resident inputs and preallocated outputs
    if uniform:
        m, n = sizes[0]
        k = min(m, n)
        A_h = torch.from_numpy(np.stack(host)).pin_memory()
        A = A_h.to(dev)
        out = (torch.empty(B, k, device=dev, dtype=torch.float64), torch.empty(B, k, m, device=dev, dtype=torch.float64),
               torch.empty(B, k, n, device=dev, dtype=torch.float64))
        call = lambda X: wc.svd_batched(X, out=out, return_info=True)
        in_bytes = A.numel() * 8
        out_bytes = sum(t.numel() for t in out) * 8
    else:
        A_h = [torch.from_numpy(a).pin_memory() for a in host]
        A = [a.to(dev) for a in A_h]
        call = lambda X: wc.svd_batched(X, return_info=True)
        in_bytes = sum(a.numel() for a in A) * 8
        out_bytes = sum(min(mm, nn) * (1 + mm + nn) for (mm, nn) in sizes) * 8
    del host
    stream = torch.cuda.current_stream()

    # warm-up (also yields sweeps per matrix for the algorithmic flop count)
    for _ in range(args.warmup):
        res = call(A)
    torch.cuda.synchronize()
    info = res[3].cpu().numpy()
    flops_alg = float(sum(workloads.f_tb(mm, nn) * max(int(s), 0) for (mm, nn), s in zip(sizes, info)))

    # ---- timed region: device-resident inputs ----
    def barrier():
        if world > 1:
            import torch.distributed as dist
            dist.barrier()
        torch.cuda.synchronize()

    barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local_dev) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            res = call(A)
        ev1.record(stream)
        barrier()
    ms = ev0.elapsed_time(ev1)
    if world > 1:
        import torch.distributed as dist
        t = torch.tensor([ms], dtype=torch.float64, device=dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / args.steps
    value = world * B * args.steps / (ms * 1e-3)

    # ---- e2e: the public end-to-end call with HOST buffers (wcsvd_batched_host): pinned inputs ->
    # H2D -> kernels -> D2H of S, U, V, pipelined over chunks inside the library; inside the timing ----
    if uniform:
        k_ = min(sizes[0])
        S_h = torch.empty(B, k_, dtype=torch.float64).pin_memory()
        U_h = torch.empty(B, k_, sizes[0][0], dtype=torch.float64).pin_memory()
        V_h = torch.empty(B, k_, sizes[0][1], dtype=torch.float64).pin_memory()

        def e2e_step():
            wc.svd_batched_host(A_h, out=(S_h, U_h, V_h))
    else:
        ks_ = [min(mm, nn) for (mm, nn) in sizes]
        out_h = ([torch.empty(k, dtype=torch.float64).pin_memory() for k in ks_],
                 [torch.empty(k, mm, dtype=torch.float64).pin_memory() for k, (mm, _) in zip(ks_, sizes)],
                 [torch.empty(k, nn, dtype=torch.float64).pin_memory() for k, (_, nn) in zip(ks_, sizes)])

        def e2e_step():
            wc.svd_batched_host(A_h, out=out_h)
    e2e_step()
    barrier()
    ee0 = torch.cuda.Event(enable_timing=True)
    ee1 = torch.cuda.Event(enable_timing=True)
    e_steps = max(1, min(args.steps, 5))
    ee0.record(stream)
    for _ in range(e_steps):
        e2e_step()
    ee1.record(stream)
    barrier()
    e_ms = ee0.elapsed_time(ee1)
    if world > 1:
        import torch.distributed as dist
        t = torch.tensor([e_ms], dtype=torch.float64, device=dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e_ms = float(t.item())
    e2e_value = world * B * e_steps / (e_ms * 1e-3)

    # plan summary: kernels launched per step = one per plan bucket + the completion pass
    plans = {}
    for (mm, nn) in set(sizes):
        p = wc.plan(mm, nn)
        plans[(p["path"], p["variant"])] = p
    launches_per_step = len(plans) + 1
    if all(p["path"] == wc.PATH_L0 for p in plans.values()):
        dominant = "l0tp_kernel" if any(p["variant"] in wc.L0_TWO_PHASE_VARIANTS for p in plans.values()) \
            else "l0_jacobi_kernel"
    else:
        dominant = "l1_gram_kernel"

    # roofline of the dominant kernel: algorithmic (textbook, sweep-normalised) flops per launch /
    # launch time. The step is one launch of it plus the tiny completion pass (ncu share in profiles/).
    achieved_tf = flops_alg / (ms_step * 1e-3) / 1e12
    prof = os.path.join(ROOT, "profiles", "ncu_summary.json")
    traffic = None
    if os.path.exists(prof):  # ncu --set full dram bytes of the same kernel (profiles/), per matrix x batch
        try:
            per = json.load(open(prof)).get(args.config, {}).get("dram_bytes_per_matrix")
            traffic = None if per is None else per * B
        except Exception:
            traffic = None
    roofline = {"bound": "alu" if dominant.startswith("l0") else "tensor", "achieved": achieved_tf,
                "peak": FP64_PEAK_NOMINAL_TFLOPS, "unit": "TFLOP/s", "frac": achieved_tf / FP64_PEAK_NOMINAL_TFLOPS,
                "traffic": traffic, "kernel": dominant,
                "algorithmic_bytes": in_bytes + out_bytes,
                "peak_note": "FP64: 148 SM x 64 FMA/clk x 2 x 1.965 GHz (MEASURED_PEAKS.json has no fp64 entry; "
                             "measured DFMA 36.5 / DMMA 37.1 TF/s, profiles/peaks_fp64_r01.json)",
                "flops": "textbook F_tb(M,N)=N(N-1)/2(8M+6N) x sweeps used, summed over the batch"}

    line = {"metric": METRIC, "value": value, "unit": "matrices/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.config}: {base.description}", "batch_per_gpu": B,
                       "sizes": f"{sizes[0][0]}x{sizes[0][1]}" if uniform else "mixed",
                       "parallelism": f"batch-parallel x{world} (weak: {B} matrices per GPU)",
                       "l2": f"inputs larger than L2 ({in_bytes / 1e6:.0f} MB per GPU vs 126 MB)"
                       if in_bytes > 126e6 else f"inputs {in_bytes / 1e6:.1f} MB fit L2; no flush",
                       "gen_seconds": round(gen_s, 2)},
            "sweeps": {"mean": float(np.mean(info)), "min": int(info.min()), "max": int(info.max())},
            "sweep_normalised_tflops": achieved_tf,
            "e2e": {"value": e2e_value, "unit": "matrices/s", "h2d_bytes_per_step": int(in_bytes),
                    "d2h_bytes_per_step": int(out_bytes)},
            "gpu_launches": launches_per_step * args.steps,
            "clocks": clk.summary(),
            "roofline": roofline}
    if rank == 0 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(args.config, idx, make, sample=args.cpu_sample)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
