"""Parity metrics between an SVD under test and the oracle -- TEST INFRASTRUCTURE ONLY.

Acceptance bars are north_star's (BASELINE.json) as restated in SURVEY.md §8(c):
  sigma:          max_i |s_i - s_ref_i| / s_ref_1                      <= 1e-12
  reconstruction: ||A - U diag(S) V^T||_F / ||A||_F                     <= 1e-12
  orthogonality:  max(max|U^T U - I|, max|V^T V - I|)                  <= 1e-11
  vectors (Z25):  clusters = maximal runs of consecutive s_ref with adjacent gaps < 1e-6 s_ref_1;
                  singleton i: |u_i . u_ref_i| >= 1 - 1e-10 and |v_i . v_ref_i| >= 1 - 1e-10;
                  cluster: ||P - P_ref||_2 <= 1e-8 for the projectors onto the cluster spans.
                  Reading R-VEC: a vector / subspace is only determined to
                  theta ~ u s_1 / delta (Wedin), delta = the gap to the other singular values and, for
                  the factor with more rows than k (U if m > n, V if m < n), also the smallest sigma of
                  the group itself (its left/right null space is the competing subspace). Where that
                  bound is looser, the bars become theta_max = 64 u s_1 / delta (projector) and
                  theta_max^2 (1 - |cos|); elsewhere north_star's 1e-10 / 1e-8 stand.
Residual and orthogonality are evaluated in numpy.longdouble for min(m,n) <= 128, else in float64
(whose own evaluation error, ~sqrt(n) 2^-53 ~ 1e-14, is 100x below the bars).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

SIGMA_TOL = 1e-12
RESID_TOL = 1e-12
ORTHO_TOL = 1e-11
VEC_TOL = 1e-10
PROJ_TOL = 1e-8
GAP_REL = 1e-6


@dataclass
class Parity:
    sigma_err: float
    resid: float
    ortho: float
    vec_err: float  # max over singletons of 1 - |cos| (scaled by the R-VEC bound where looser)
    proj_err: float  # max over clusters of ||P - P_ref||_2 (scaled likewise)
    n_clusters: int
    notes: list = field(default_factory=list)

    def ok(self, sigma_tol=SIGMA_TOL, resid_tol=RESID_TOL, ortho_tol=ORTHO_TOL,
           vec_tol=VEC_TOL, proj_tol=PROJ_TOL) -> bool:
        return (self.sigma_err <= sigma_tol and self.resid <= resid_tol and self.ortho <= ortho_tol
                and self.vec_err <= vec_tol and self.proj_err <= proj_tol)

    def as_dict(self):
        return dict(sigma_err=self.sigma_err, resid=self.resid, ortho=self.ortho, vec_err=self.vec_err,
                    proj_err=self.proj_err, n_clusters=self.n_clusters)


def clusters(s_ref: np.ndarray, gap_rel: float = GAP_REL) -> list:
    """Maximal runs of consecutive sorted singular values whose adjacent gaps are < gap_rel*s_1."""
    k = len(s_ref)
    if k == 0:
        return []
    s1 = s_ref[0] if s_ref[0] > 0 else 1.0
    out, start = [], 0
    for i in range(1, k):
        if s_ref[i - 1] - s_ref[i] >= gap_rel * s1:
            out.append((start, i))
            start = i
    out.append((start, k))
    return out


def residual(A, S, U, V) -> float:
    k = len(S)
    small = k <= 128
    dt = np.longdouble if small else np.float64
    A_ = np.asarray(A, dtype=dt)
    R = A_ - (np.asarray(U, dtype=dt) * np.asarray(S, dtype=dt)) @ np.asarray(V, dtype=dt).T
    nA = np.sqrt((A_ * A_).sum())
    nR = np.sqrt((R * R).sum())
    return float(nR / nA) if nA > 0 else float(nR)


def orthogonality(Q) -> float:
    k = Q.shape[1]
    dt = np.longdouble if k <= 128 else np.float64
    Q_ = np.asarray(Q, dtype=dt)
    return float(np.abs(Q_.T @ Q_ - np.eye(k, dtype=dt)).max()) if k else 0.0


# fp32 (north_star gives sigma / residual / orthogonality only; the vector floors follow from a backward
# error of ~1e-6 ||A|| after ~300 fp32 rotations per column: angle ~1e-3 at relative gaps ~1e-3).
FP32_BARS = dict(sigma_tol=1e-5, resid_tol=1e-5, ortho_tol=1e-4, vec_tol=1e-5, proj_tol=1e-3)


def compare(A, S, U, V, S_ref, U_ref, V_ref, check_vectors: bool = True, u: float = 2.0 ** -53,
            vec_tol: float = VEC_TOL, proj_tol: float = PROJ_TOL) -> Parity:
    """u: unit roundoff of the arithmetic under test (2^-53 fp64, 2^-24 fp32) for the R-VEC bound;
    vec_tol / proj_tol: the floors the returned errors are scaled against (Parity.ok() bars)."""
    A = np.asarray(A, dtype=np.float64)
    S = np.asarray(S, dtype=np.float64)
    S_ref = np.asarray(S_ref, dtype=np.float64)
    s1 = S_ref[0] if len(S_ref) and S_ref[0] > 0 else 1.0
    sig = float(np.abs(S - S_ref).max() / s1) if len(S) else 0.0
    res = residual(A, S, U, V) if U is not None and V is not None else 0.0
    orth = 0.0
    if U is not None:
        orth = max(orth, orthogonality(U))
    if V is not None:
        orth = max(orth, orthogonality(V))
    vec_err, proj_err, ncl = 0.0, 0.0, 0
    if check_vectors and U is not None and V is not None:
        k = len(S_ref)
        for (a, b) in clusters(S_ref):
            gap = np.inf
            if a > 0:
                gap = min(gap, S_ref[a - 1] - S_ref[a])
            if b < k:
                gap = min(gap, S_ref[b - 1] - S_ref[b])
            if b - a > 1:
                ncl += 1
            for (X, Xr) in ((U, U_ref), (V, V_ref)):
                delta = gap
                if X.shape[0] > k:  # the long factor: its null space competes (Wedin)
                    delta = min(delta, S_ref[b - 1])
                theta = 64 * u * s1 / delta if delta > 0 else np.inf
                if b - a == 1:
                    c = abs(float(np.dot(X[:, a], Xr[:, a])))
                    vec_err = max(vec_err, (1.0 - c) / max(1.0, theta ** 2 / vec_tol))
                else:
                    P = X[:, a:b] @ X[:, a:b].T
                    Pr = Xr[:, a:b] @ Xr[:, a:b].T
                    e = float(np.linalg.norm(P - Pr, 2))
                    proj_err = max(proj_err, e / max(1.0, theta / proj_tol))
    return Parity(sig, res, orth, vec_err, proj_err, ncl)
