"""Pins of the CPU oracle against things other than itself.

Each test is chosen so that a plausible mistake in oracle/oracle_body.inc (a dropped term, a wrong
sign in eq (3)/(4), a transposed operand, a missed un-orientation) fails at least one of them.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
from oracle import compare
import workloads

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
U53 = 2.0 ** -53


def test_long_double_is_x87():
    # The oracle's parity precision relies on the 64-bit mantissa.
    assert oracle.ldbl_mant_dig() == 64


@pytest.mark.parametrize("case", json.load(open(os.path.join(GOLDEN, "svd_closed_forms.json")))["cases"],
                         ids=lambda c: c["name"])
def test_golden_closed_forms(case):
    A = np.array(case["A"], dtype=np.float64)
    S_exp = np.array([eval(s, {"sqrt": math.sqrt}) for s in case["S"]])
    r = oracle.svd(A)
    assert r.converged
    assert np.allclose(r.S, S_exp, rtol=0, atol=4 * U53 * S_exp[0])
    if "sweeps" in case:
        assert r.sweeps == case["sweeps"]
    if "V_abs" in case:
        assert np.allclose(np.abs(r.V), np.array(case["V_abs"]), atol=4 * U53)


def _closed_2x2(a, b, c, d):
    # P1: sigma_{1,2} = (sqrt((a+d)^2+(c-b)^2) +- sqrt((a-d)^2+(b+c)^2)) / 2, |.| for sigma_2.
    p = math.sqrt((a + d) ** 2 + (c - b) ** 2)
    q = math.sqrt((a - d) ** 2 + (b + c) ** 2)
    return (p + q) / 2, abs(p - q) / 2


def test_p1_2x2_closed_form():
    rng = np.random.default_rng(11)
    for _ in range(200):
        a, b, c, d = rng.standard_normal(4)
        r = oracle.svd(np.array([[a, b], [c, d]]))
        s1, s2 = _closed_2x2(a, b, c, d)
        assert abs(r.S[0] - s1) <= 8 * U53 * s1
        assert abs(r.S[1] - s2) <= 8 * U53 * s1


def test_p3_two_sided_2x2_zeroes_offdiagonal():
    # §II.D: one Givens step with rho as printed diagonalises a 2x2 symmetric B.
    rng = np.random.default_rng(12)
    for _ in range(50):
        X = rng.standard_normal((2, 2))
        B = X + X.T
        lam, J, sw = oracle.syevj(B)
        assert sw >= 1
        D = J.T @ B @ J
        assert abs(D[0, 1]) <= 8 * U53 * np.abs(B).max()
        assert np.allclose(np.sort(lam), np.linalg.eigvalsh(B), atol=8 * U53 * np.abs(B).max())


def test_syevj_vs_lapack_eigvalsh():
    rng = np.random.default_rng(13)
    for n in (4, 16, 32, 64):
        X = rng.standard_normal((n + 3, n))
        B = X.T @ X
        lam, J, sw = oracle.syevj(B)
        assert sw > 0
        ev = np.linalg.eigvalsh(B)
        assert np.abs(np.sort(lam) - ev).max() <= 64 * U53 * ev[-1]
        assert np.abs(J.T @ J - np.eye(n)).max() <= 16 * U53
        assert np.abs(J.T @ B @ J - np.diag(lam)).max() <= 64 * U53 * ev[-1]


def test_p7_diagonal_and_permuted_diagonal():
    d = np.array([0.5, -3.0, 2.0, 1.0, -0.25])
    A = np.diag(d)
    r = oracle.svd(A)
    assert r.sweeps == 1 and r.rotations == 0
    assert np.array_equal(r.S, np.sort(np.abs(d))[::-1])
    for X in (r.U, r.V):
        assert set(np.unique(np.abs(X))) <= {0.0, 1.0}
    assert np.array_equal((r.U * r.S) @ r.V.T, A)
    # permuted, rectangular, both orientations
    rng = np.random.default_rng(7)
    P = np.zeros((7, 4))
    rows = rng.permutation(7)[:4]
    vals = np.array([1.5, -4.0, 0.75, 2.5])
    for j in range(4):
        P[rows[j], j] = vals[j]
    for X in (P, P.T):
        r = oracle.svd(X)
        assert r.sweeps == 1
        assert np.array_equal(r.S, np.sort(np.abs(vals))[::-1])
        assert np.array_equal((r.U * r.S) @ r.V.T, X)


@pytest.mark.parametrize("kappa", [1e1, 1e4, 1e8, 1e12])
def test_p8_prescribed_spectrum(kappa):
    # A = Q1 diag(s) Q2^T: sigma = s to c*u*s_1 absolute (rounding A to fp64 already moves sigma by ~u s_1).
    rng = workloads.matrix_rng(901, int(np.log10(kappa)))
    for (m, n) in ((32, 32), (48, 20), (20, 48)):
        k = min(m, n)
        s = kappa ** (-np.arange(k) / (k - 1))
        A = workloads.prescribed(rng, m, n, s)
        r = oracle.svd(A)
        assert r.converged
        assert np.abs(r.S - s).max() <= 20 * U53 * s[0]


def test_p9_invariants():
    rng = np.random.default_rng(21)
    for (m, n) in ((40, 24), (24, 40), (64, 64), (100, 3), (3, 100)):
        A = rng.standard_normal((m, n))
        r = oracle.svd(A)
        fro2 = np.sum(np.asarray(A, np.longdouble) ** 2)
        assert abs(np.sum(np.asarray(r.S, np.longdouble) ** 2) - fro2) / fro2 <= 8 * U53
        assert compare.orthogonality(r.U) <= 4 * U53
        assert compare.orthogonality(r.V) <= 4 * U53
        assert compare.residual(A, r.S, r.U, r.V) <= 8 * U53
        assert np.all(np.diff(r.S) <= 0)


def test_p6_brute_force_eigenvalues_of_gram():
    rng = np.random.default_rng(31)
    # n <= 3: characteristic polynomial of A^T A solved in closed form (trigonometric cubic)
    for _ in range(50):
        A = rng.standard_normal((5, 3))
        G = A.T @ A
        p1 = G[0, 1] ** 2 + G[0, 2] ** 2 + G[1, 2] ** 2
        q = np.trace(G) / 3
        p2 = (G[0, 0] - q) ** 2 + (G[1, 1] - q) ** 2 + (G[2, 2] - q) ** 2 + 2 * p1
        p = math.sqrt(p2 / 6)
        Bm = (G - q * np.eye(3)) / p
        rr = np.clip(np.linalg.det(Bm) / 2, -1, 1)
        phi = math.acos(rr) / 3
        e1 = q + 2 * p * math.cos(phi)
        e3 = q + 2 * p * math.cos(phi + 2 * math.pi / 3)
        e2 = 3 * q - e1 - e3
        r = oracle.svd(A)
        assert np.allclose(r.S ** 2, [e1, e2, e3], rtol=0, atol=1e-12 * e1)
    # larger: eigvalsh of the Gram (library routine) and LAPACK svd
    for (m, n) in ((64, 64), (50, 30), (30, 50)):
        A = rng.standard_normal((m, n))
        r = oracle.svd(A)
        ev = np.sort(np.linalg.eigvalsh(A.T @ A if m >= n else A @ A.T))[::-1]
        assert np.abs(r.S ** 2 - ev).max() <= 1e-12 * ev[0]
        s = np.linalg.svd(A, compute_uv=False)
        assert np.abs(r.S - s).max() <= 64 * U53 * s[0]


def test_p10_power_of_two_scaling_is_bitwise():
    rng = np.random.default_rng(41)
    A = rng.standard_normal((24, 17))
    r0 = oracle.svd(A)
    for e in (-37, 5, 300):
        r = oracle.svd(A * 2.0 ** e)
        assert np.array_equal(r.U, r0.U) and np.array_equal(r.V, r0.V)
        assert np.array_equal(r.S, r0.S * 2.0 ** e)
        assert r.sweeps == r0.sweeps


def test_p11_transpose_symmetry_is_bitwise():
    rng = np.random.default_rng(42)
    for (m, n) in ((24, 17), (17, 24), (16, 16)):
        A = rng.standard_normal((m, n))
        r = oracle.svd(A)
        rt = oracle.svd(A.T.copy())
        if m != n:
            assert np.array_equal(r.S, rt.S)
            assert np.array_equal(r.U, rt.V) and np.array_equal(r.V, rt.U)
        else:  # square: both orientations iterate on A itself vs A^T; only S is fixed
            assert np.abs(r.S - rt.S).max() <= 8 * U53 * r.S[0]


def test_z15_sign_rule_fixes_the_square_factor():
    # Z15 (oracle step 8): singular vectors are unique only up to a joint sign; the sign rule (largest-|.|
    # entry of each square-factor column positive, first on ties) makes them a function of A alone. Pin:
    # permuting the columns of a tall A (A P = U S (P^T V)^T) must return P^T V and the same U without
    # any sign alignment, and permuting the rows of a wide A (P A = (P U) S V^T) must return P U and the
    # same V -- the Jacobi iteration on the permuted matrix takes a different rotation sequence, so only
    # the rule (applied to the right factor, on the right entry) can make the signs agree.
    rng = np.random.default_rng(52)
    for (m, n) in ((30, 12), (12, 30)):
        A = workloads.prescribed(rng, m, n, np.geomspace(1.0, 1e-2, min(m, n)))  # well-separated sigma
        r = oracle.svd(A)
        if m >= n:
            p = rng.permutation(n)
            rp = oracle.svd(A[:, p].copy())
            Vexp, Uexp = r.V[p, :], r.U
            assert np.abs(rp.V - Vexp).max() <= 1e-12 and np.abs(rp.U - Uexp).max() <= 1e-12
        else:
            p = rng.permutation(m)
            rp = oracle.svd(A[p, :].copy())
            Uexp, Vexp = r.U[p, :], r.V
            assert np.abs(rp.U - Uexp).max() <= 1e-12 and np.abs(rp.V - Vexp).max() <= 1e-12
        assert np.abs(rp.S - r.S).max() <= 8 * U53 * r.S[0]
        # and the rule itself: every square-factor column's largest-|.| entry (first on ties) is > 0
        Q = rp.V if m >= n else rp.U
        assert all(Q[np.argmax(np.abs(Q[:, j])), j] > 0 for j in range(Q.shape[1]))


def test_z14_rank_deficient_completion():
    rng = np.random.default_rng(51)
    # exact zero columns, and an exactly rank-2 product
    A = rng.standard_normal((8, 5))
    A[:, 1] = 0
    A[:, 3] = 0
    r = oracle.svd(A)
    assert r.S[-1] == 0 and r.S[-2] == 0
    assert compare.orthogonality(r.U) <= 4 * U53
    assert compare.residual(A, r.S, r.U, r.V) <= 8 * U53
    Z = np.zeros((6, 4))
    r = oracle.svd(Z)
    assert np.all(r.S == 0)
    assert compare.orthogonality(r.U) == 0 and compare.orthogonality(r.V) == 0
    X = rng.standard_normal((10, 2)) @ rng.standard_normal((2, 7))
    r = oracle.svd(X)
    assert r.S[2] <= 1e-14 * r.S[0]
    assert compare.orthogonality(r.U) <= 8 * U53
    assert compare.residual(X, r.S, r.U, r.V) <= 16 * U53


def test_max_sweeps_not_converged_is_finite():
    A = np.random.default_rng(61).standard_normal((32, 32))
    r = oracle.svd(A, max_sweeps=1)
    assert not r.converged and r.sweeps == 1
    assert np.all(np.isfinite(r.S)) and np.all(np.isfinite(r.U)) and np.all(np.isfinite(r.V))


def test_sweep_counts_in_expected_range():
    # P15 sanity range (not parity): long-double row-cyclic 9-11 sweeps on Gaussian 24..64.
    rng = np.random.default_rng(71)
    for n in (24, 32, 64):
        r = oracle.svd(rng.standard_normal((n, n)))
        assert 7 <= r.sweeps <= 13


def test_batch_matches_single_and_double_instantiation():
    cfg = workloads.get_config("C1", batch=10)
    As = cfg.matrices()
    S, U, V, info = oracle.svd_batch(As)
    for k, A in enumerate(As):
        r = oracle.svd(A)
        assert np.array_equal(S[k], r.S) and np.array_equal(U[k], r.U) and info[k] == r.sweeps
    Sd, Ud, Vd, infod = oracle.svd_batch(As, precision="d")
    for k, A in enumerate(As):
        p = compare.compare(A, Sd[k], Ud[k], Vd[k], S[k], U[k], V[k])
        assert p.sigma_err <= 1e-13 and p.resid <= 1e-13 and p.ortho <= 1e-13


def test_compare_metrics_detect_errors():
    # The parity metric itself must flag a wrong sigma, a non-orthogonal U and a swapped vector.
    A = np.random.default_rng(81).standard_normal((12, 8))
    r = oracle.svd(A)
    assert compare.compare(A, r.S, r.U, r.V, r.S, r.U, r.V).ok()
    S2 = r.S.copy(); S2[3] *= 1 + 1e-9
    assert not compare.compare(A, S2, r.U, r.V, r.S, r.U, r.V).ok()
    U2 = r.U.copy(); U2[:, [1, 2]] = U2[:, [2, 1]]
    assert not compare.compare(A, r.S, U2, r.V, r.S, r.U, r.V).ok()
    assert compare.compare(A, r.S, -r.U, -r.V, r.S, r.U, r.V).ok()  # joint sign is free


def test_c1_workload_spectrum_matches_prescription():
    # Input recipe check: C1 matrices carry the prescribed s (oracle agrees to ~u s_1).
    cfg = workloads.get_config("C1", batch=5)
    for k in range(5):
        r = oracle.svd(cfg.make(k))
        assert np.abs(r.S - cfg.spectrum(k)).max() <= 20 * U53


def test_oracle_table7_standins(capsys):
    # the Table VII stand-ins (sizes and condition numbers of the paper's picks,
    # PAPER.md:469-476; kappa 3.1 .. 8.08e15) -- pinned to their prescribed spectra (known by
    # construction, exact up to the fp64 rounding of A) and to the invariants; the sweep counts are
    # printed as the reference column of the GPU robustness table (tools/robustness.py).
    cfg = workloads.table7_config()
    mats = cfg.matrices()
    S, U, V, info = oracle.svd_batch(mats)
    for k, A in enumerate(mats):
        s_true = cfg.spectrum(k)
        assert info[k] > 0
        assert np.abs(S[k] - s_true).max() <= 1e-13
        # north_star's bars (the residual is formed in fp64 from fp64-rounded factors)
        assert compare.residual(A, S[k], U[k], V[k]) <= 1e-12
        assert compare.orthogonality(U[k]) <= 1e-11 and compare.orthogonality(V[k]) <= 1e-11
    with capsys.disabled():
        print("\noracle sweeps on the Table VII stand-ins:",
              {workloads.TABLE7[k][0]: int(info[k]) for k in range(len(mats))})
