"""Parity of the Level-1 Gram path (Gram -> EVD -> DMMA update -> off-norm test; Alg 1 / Alg 2
l.10-11) with the oracle, on ragged shapes and the C3/C4 workloads."""
import numpy as np
import pytest

import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
from tests.gpu_helpers import check_parity, gpu_svd_list, gpu_svd_tensor

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("shapes", [
    [(97, 97), (128, 128), (130, 99), (99, 130), (200, 120)],
    [(256, 256), (300, 170), (170, 300), (1024, 100), (100, 1024)],
    [(513, 257), (600, 600)],
])
def test_l1_ragged_shapes(shapes):
    mats = [workloads.gaussian(workloads.matrix_rng(500 + i, 3), m, n) for i, (m, n) in enumerate(shapes)]
    for (m, n) in shapes:
        assert wc.plan(m, n)["path"] == wc.PATH_GRAM
    S, U, V, info = gpu_svd_list(mats)
    check_parity(mats, S, U, V, info)


@pytest.mark.parametrize("w", [8, 16])
def test_l1_forced_on_small_shapes(w):
    # The Gram path on shapes the planner would give to Level 0 (ragged tails, m<n, tiny).
    shapes = [(64, 64), (40, 24), (24, 40), (17, 9), (33, 65), (5, 3)]
    mats = [workloads.gaussian(workloads.matrix_rng(520 + i, w), m, n) for i, (m, n) in enumerate(shapes)]
    S, U, V, info = gpu_svd_list(mats, force_path=wc.PATH_GRAM, force_w=w)
    check_parity(mats, S, U, V, info)


def test_l1_ill_conditioned_and_rank_deficient():
    rng = workloads.matrix_rng(530, 0)
    mats = []
    for kappa in (1e6, 1e12):
        s = kappa ** (-np.arange(150) / 149.0)
        mats.append(workloads.prescribed(rng, 200, 150, s))
    Z = workloads.gaussian(rng, 180, 130)
    Z[:, 5] = 0.0
    Z[:, 77] = 0.0
    mats.append(Z)
    mats.append(workloads.gaussian(rng, 150, 3) @ workloads.gaussian(rng, 3, 140))
    S, U, V, info = gpu_svd_list(mats)
    check_parity(mats, S, U, V, info)


def test_c3_sampled():
    cfg = workloads.get_config("C3", batch=256)
    mats = cfg.matrices()
    S, U, V, info = gpu_svd_tensor(np.stack(mats))
    assert np.all(info > 0)
    check_parity(mats, S, U, V, info, idx=list(range(0, 256, 8)))  # 32 of 256 against the oracle


def test_c4_sampled():
    cfg = workloads.get_config("C4", batch=64)
    mats = cfg.matrices()
    S, U, V, info = gpu_svd_tensor(np.stack(mats))
    assert np.all(info > 0)
    check_parity(mats, S, U, V, info, idx=list(range(0, 64, 4)))  # 16 of 64 against the oracle
    for k in range(0, 64, 4):
        assert np.abs(S[k] - cfg.spectrum(k)).max() <= 1e-13


def test_l1_1024_rows_against_the_oracle():
    # M = 1024 (the largest dimension the boundary accepts) against the long-double oracle itself, not
    # only LAPACK sigma: a 1024 x 256 and its transpose (seconds in the oracle; 1024^2 takes minutes)
    shapes = [(1024, 256), (256, 1024)]
    mats = [workloads.gaussian(workloads.matrix_rng(545, i), m, n) for i, (m, n) in enumerate(shapes)]
    S, U, V, info = gpu_svd_list(mats)
    check_parity(mats, S, U, V, info)


def test_l1_1024_square_against_the_oracle():
    # the largest size of the boundary against the long-double oracle itself (~2 min of oracle time
    # on one host core; tools/oracle_check_large.py runs three such matrices)
    cfg = workloads.get_config("C5", batch=1)
    mats = [cfg.make(0)]
    assert mats[0].shape == (1024, 1024)
    S, U, V, info = gpu_svd_list(mats)
    check_parity(mats, S, U, V, info)


def test_l1_bitwise_deterministic_across_batch_composition():
    mats = [workloads.gaussian(workloads.matrix_rng(540, i), 160, 140) for i in range(6)]
    S1, U1, V1, _ = gpu_svd_list(mats)
    S2, U2, V2, _ = gpu_svd_list([mats[3]] + [workloads.gaussian(workloads.matrix_rng(541, 0), 300, 200)])
    assert np.array_equal(S1[3], S2[0]) and np.array_equal(U1[3], U2[0]) and np.array_equal(V1[3], V2[0])


@pytest.mark.parametrize("w", [8, 16])
def test_wcycle_forced(w):
    # W-cycle recursion (Alg 2 l.12-14): Level-1 super-blocks w1 = 64 -> Level-2 EVD width w2 = w.
    shapes = [(256, 256), (300, 200), (200, 300), (1024, 130), (150, 140), (130, 129)]
    mats = [workloads.gaussian(workloads.matrix_rng(550 + i, w), m, n) for i, (m, n) in enumerate(shapes)]
    for (m, n) in shapes:
        p = wc.plan(m, n, force_path=wc.PATH_WCYCLE, force_w=w)
        assert p["path"] == wc.PATH_WCYCLE and p["w"] == 64 and p["w2"] == w
    S, U, V, info = gpu_svd_list(mats, force_path=wc.PATH_WCYCLE, force_w=w)
    check_parity(mats, S, U, V, info)


def test_wcycle_ill_conditioned():
    rng = workloads.matrix_rng(560, 0)
    s = 1e10 ** (-np.arange(200) / 199.0)
    mats = [workloads.prescribed(rng, 260, 200, s)]
    S, U, V, info = gpu_svd_list(mats, force_path=wc.PATH_WCYCLE)
    check_parity(mats, S, U, V, info)


def test_c5_mixed_sampled_and_1024_properties():
    # C5 mixed sizes (first 201 matrices incl. k = 0, 100, 200 forced to 1024x1024): oracle parity on
    # the matrices with min(m, n) <= 160 (seconds in long double), and for the 1024^2 ones the
    # size-independent properties plus LAPACK sigma.
    cfg = workloads.get_config("C5", batch=201)
    mats = cfg.matrices()
    S, U, V, info = gpu_svd_list(mats)
    assert np.all(info > 0)
    small = [k for k, (m, n) in enumerate(cfg.sizes) if min(m, n) <= 160][:12]
    check_parity(mats, S, U, V, info, idx=small)
    from oracle import compare
    for k in (0, 100, 200):
        A = mats[k]
        assert compare.residual(A, S[k], U[k], V[k]) <= 1e-12
        assert compare.orthogonality(U[k]) <= 1e-11 and compare.orthogonality(V[k]) <= 1e-11
        s_ref = np.linalg.svd(A, compute_uv=False)
        assert np.abs(S[k] - s_ref).max() / s_ref[0] <= 1e-12


def test_removed_split_executor_is_rejected():
    # wcsvd_opts.pair_warps = 2 (round-1 ablation executor) was removed: -12 before anything is enqueued
    import torch
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wcm
    A = torch.from_numpy(workloads.gaussian(workloads.matrix_rng(570, 2), 256, 256)).cuda()[None]
    with pytest.raises(wcm.WcsvdError) as ei:
        wcm.svd_batched(A, pair_warps=2)
    assert ei.value.code == -12


@pytest.mark.parametrize("shapes", [
    [(256, 256), (300, 170), (170, 300), (1024, 128), (97, 97), (513, 257)],
    [(64, 64), (40, 33), (33, 65)],
])
def test_panel_path_group_i(shapes):
    # group (i) (Alg 2 l.8-9): J from one-sided Jacobi of the CholeskyQR-compressed pair panel
    mats = [workloads.gaussian(workloads.matrix_rng(590 + i, 9), m, n) for i, (m, n) in enumerate(shapes)]
    for (m, n) in shapes:
        assert wc.plan(m, n, force_path=wc.PATH_PANEL)["path"] == wc.PATH_PANEL
    S, U, V, info = gpu_svd_list(mats, force_path=wc.PATH_PANEL)
    check_parity(mats, S, U, V, info)


def test_panel_path_ill_conditioned_falls_back_per_pair():
    # nearly dependent / rank-deficient panels take the two-sided EVD for that pair (tiny Cholesky pivot)
    rng = workloads.matrix_rng(595, 0)
    s = 1e12 ** (-np.arange(150) / 149.0)
    A1 = workloads.prescribed(rng, 200, 150, s)
    Z = workloads.gaussian(rng, 180, 130)
    Z[:, 5] = 0.0
    Z[:, 77] = Z[:, 3]
    mats = [A1, Z]
    S, U, V, info = gpu_svd_list(mats, force_path=wc.PATH_PANEL)
    check_parity(mats, S, U, V, info)
