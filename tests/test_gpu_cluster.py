"""Tailoring: a Gram-path matrix spread over a thread-block
cluster of 2, 4 or 8 CTAs (dataflow counters, votes and finalisation arrays in rank 0's distributed
shared memory). The pairs' arithmetic is unchanged, so every output must be BITWISE equal to the
one-CTA kernel, and the planner-chosen cluster (small batches of large matrices) must match the oracle."""
import numpy as np
import pytest

import workloads
from tests.gpu_helpers import check_parity, gpu_svd_list

pytestmark = pytest.mark.gpu

SHAPES = [(1024, 1024), (700, 1000), (513, 257), (256, 256), (130, 99), (1000, 300)]


def _mats(shapes, seed):
    return [workloads.gaussian(workloads.matrix_rng(seed, k), m, n) for k, (m, n) in enumerate(shapes)]


def test_cluster_sizes_bitwise_equal():
    mats = _mats(SHAPES, 610)
    ref = gpu_svd_list(mats, cluster_ctas=1)
    for cl in (2, 4, 8):
        out = gpu_svd_list(mats, cluster_ctas=cl)
        for k in range(len(mats)):
            for a, b in zip(ref[:3], out[:3]):
                assert np.array_equal(a[k], b[k]), (cl, k, mats[k].shape)
            assert ref[3][k] == out[3][k]


def test_planner_cluster_small_batch_parity():
    # two large matrices: the planner spreads each over a cluster (tailoring); parity with the oracle
    mats = _mats([(1024, 1024), (900, 640)], 611)
    S, U, V, info = gpu_svd_list(mats)
    check_parity(mats, S, U, V, info)
    ref = gpu_svd_list(mats, cluster_ctas=1)
    for k in range(2):
        assert np.array_equal(S[k], ref[0][k]) and np.array_equal(U[k], ref[1][k]) and np.array_equal(V[k], ref[2][k])


def test_cluster_fp32_and_values_only():
    import torch
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc

    mats = _mats([(800, 512), (300, 700)], 612)
    As = [torch.from_numpy(a).cuda() for a in mats]
    S1, _, _ = wc.svd_batched(As, compute_uv=False, cluster_ctas=1)
    S4, _, _ = wc.svd_batched(As, compute_uv=False, cluster_ctas=4)
    for a, b in zip(S1, S4):
        assert torch.equal(a, b)
    Af = [a.float() for a in As]
    S1, U1, V1 = wc.svd_batched(Af, cluster_ctas=1)
    S8, U8, V8 = wc.svd_batched(Af, cluster_ctas=8)
    for k in range(2):
        assert torch.equal(S1[k], S8[k]) and torch.equal(U1[k], U8[k]) and torch.equal(V1[k], V8[k])
