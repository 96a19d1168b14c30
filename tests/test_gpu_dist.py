"""Multi-GPU path on one GPU: two ranks (gloo control plane, both on cuda:0)
factor their LPT shares of one fixed mixed batch with svd_batched_dist and gather S to rank 0; every
per-matrix output must be BITWISE equal to the single-rank call (the plan and the kernels depend on
(m, n, A) only, never on batch composition or rank count)."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import workloads

pytestmark = pytest.mark.gpu

SIZES = [(1024, 1024), (300, 200), (64, 64), (40, 500), (256, 256), (1000, 130), (33, 33), (700, 700),
         (128, 96), (90, 300), (64, 64), (512, 100)]
SEED = 4242


def _make(k):
    return workloads.gaussian(workloads.matrix_rng(SEED, k), *SIZES[k])


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, outdir):
    import torch.distributed as dist

    from paper_conf_sc_xiaopxsmmlzt22_b200 import dist as wdist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    idx, S, U, V = wdist.svd_batched_dist(SIZES, _make, rank, world)
    torch.cuda.synchronize()
    np.savez(os.path.join(outdir, f"r{rank}.npz"), idx=np.array(idx),
             **{f"S{k}": s.cpu().numpy() for k, s in zip(idx, S)},
             **{f"U{k}": u.cpu().numpy() for k, u in zip(idx, U)},
             **{f"V{k}": v.cpu().numpy() for k, v in zip(idx, V)})
    full = wdist.gather_sigma(idx, S, SIZES)
    if rank == 0:
        np.savez(os.path.join(outdir, "gathered.npz"), **{f"S{k}": s.numpy() for k, s in enumerate(full)})
    dist.barrier()
    dist.destroy_process_group()


def test_dist_world2_bitwise_equal_to_single_rank():
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
    from paper_conf_sc_xiaopxsmmlzt22_b200 import dist as wdist

    parts = wdist.lpt_partition(SIZES, 2)
    assert parts[0] and parts[1]
    mats = [torch.from_numpy(_make(k)).cuda() for k in range(len(SIZES))]
    S1, U1, V1 = wc.svd_batched(mats)
    torch.cuda.synchronize()
    with tempfile.TemporaryDirectory() as td:
        ctx = mp.get_context("spawn")
        port = _free_port()
        procs = [ctx.Process(target=_worker, args=(r, 2, port, td)) for r in range(2)]
        for p in procs:
            p.start()
        for p in procs:
            p.join(timeout=600)
            assert p.exitcode == 0
        seen = set()
        for r in range(2):
            z = np.load(os.path.join(td, f"r{r}.npz"))
            assert sorted(z["idx"].tolist()) == sorted(parts[r])
            for k in z["idx"].tolist():
                seen.add(k)
                assert np.array_equal(z[f"S{k}"], S1[k].cpu().numpy()), k
                assert np.array_equal(z[f"U{k}"], U1[k].cpu().numpy()), k
                assert np.array_equal(z[f"V{k}"], V1[k].cpu().numpy()), k
        assert seen == set(range(len(SIZES)))
        g = np.load(os.path.join(td, "gathered.npz"))
        for k in range(len(SIZES)):
            assert np.array_equal(g[f"S{k}"], S1[k].cpu().numpy()), k
