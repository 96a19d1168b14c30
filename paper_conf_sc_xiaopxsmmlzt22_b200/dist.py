"""Multi-GPU batch partition: one process per GPU, no collective on the hot path.

The matrices of a batch are independent, so the path shards with zero exchange: every rank computes
the same greedy LPT partition from the sizes alone (largest estimated cost first, each matrix to the
least-loaded rank, ties to the lower rank), factors its share with ``svd_batched`` on its own GPU,
and -- only if results are wanted on one rank -- S is gathered once after the batch through
torch.distributed (NCCL over NVLink/NVSwitch; gloo in the CPU tests). Per-matrix outputs are
bitwise independent of the rank count because the plan and the kernels depend on (m, n, A) only.
"""
from __future__ import annotations

from typing import Callable, Sequence

__all__ = ["cost", "lpt_partition", "svd_batched_dist", "gather_sigma"]


def cost(m: int, n: int) -> float:
    """Estimated work of one sweep, F_tb(M, N) = N(N-1)/2 (8M + 6N), M = max(m, n)."""
    M, N = max(m, n), min(m, n)
    return N * (N - 1) / 2.0 * (8.0 * M + 6.0 * N)


def lpt_partition(sizes: Sequence, world: int) -> list:
    """Greedy LPT: sort by cost descending (ties by index), assign to the least-loaded rank (ties to
    the lowest rank). Returns, per rank, the sorted list of batch indices it owns."""
    order = sorted(range(len(sizes)), key=lambda k: (-cost(*sizes[k]), k))
    load = [0.0] * world
    parts = [[] for _ in range(world)]
    for k in order:
        r = min(range(world), key=lambda i: (load[i], i))
        parts[r].append(k)
        load[r] += cost(*sizes[k])
    return [sorted(p) for p in parts]


def svd_batched_dist(sizes: Sequence, make_matrix: Callable[[int], "object"], rank: int, world: int,
                     device=None, **kw):
    """Factor this rank's LPT share of the batch. ``make_matrix(k)`` returns matrix k (numpy or
    torch, CPU or CUDA); each rank builds only its own matrices (no scatter). Returns
    (indices, S, U, V) for the local share."""
    import numpy as np
    import torch

    from . import svd_batched

    mine = lpt_partition(sizes, world)[rank]
    dev = device or torch.device("cuda", torch.cuda.current_device())
    mats = []
    for k in mine:
        a = make_matrix(k)
        a = torch.as_tensor(np.ascontiguousarray(a)) if not isinstance(a, torch.Tensor) else a
        mats.append(a.to(dev, dtype=torch.float64))
    if not mats:
        return mine, [], [], []
    S, U, V = svd_batched(mats, **kw)
    return mine, S, U, V


def gather_sigma(indices: list, S: list, sizes: Sequence, group=None, dst: int = 0):
    """Gather every rank's singular values to rank `dst` (one collective, after the batch).
    Returns the full list S[k] (k = 0..batch-1, CPU float64 tensors) on `dst`, None elsewhere.
    Works with any backend: the padded [rows, 1 + kmax] block (column 0 = batch index) is packed on
    the host, moved once to the backend's device (CUDA for NCCL, CPU for gloo) and gathered with one
    all_gather (plus one tiny all_gather of the row counts)."""
    import numpy as np
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    kmax = max((min(m, n) for (m, n) in sizes), default=0)
    nloc = torch.tensor([len(indices)], dtype=torch.int64, device=dev)
    counts = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(counts, nloc, group=group)
    counts = [int(c.item()) for c in counts]
    cmax = max(max(counts), 1)
    host = np.full((cmax, kmax + 1), np.nan)
    for j, (k, s) in enumerate(zip(indices, S)):
        host[j, 0] = float(k)
        sv = s.detach().cpu().numpy() if isinstance(s, torch.Tensor) else np.asarray(s)
        host[j, 1:1 + sv.size] = sv.reshape(-1)
    buf = torch.from_numpy(host).to(dev)
    outs = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(outs, buf, group=group)
    if rank != dst:
        return None
    full = [None] * len(sizes)
    for r in range(world):
        o = outs[r].cpu()
        for j in range(counts[r]):
            k = int(o[j, 0].item())
            full[k] = o[j, 1:1 + min(sizes[k])].clone()
    return full
