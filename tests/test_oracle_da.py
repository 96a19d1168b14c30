"""Pins of the data-assimilation oracle (oracle/da.py, DESIGN.md §3 R-DA) against what
the mathematics fixes: the Y = 0 and one-member closed forms, the defining identity T A T = I, and the
Sherman-Morrison-Woodbury forms of A^{-1} Y^T d and A^{-1} (a transposed Y or a dropped identity
fails them)."""
import numpy as np

from oracle import da


def _case(m, n, seed):
    rng = np.random.default_rng(seed)
    return rng.standard_normal((m, n)) / np.sqrt(n - 1 if n > 1 else 1), rng.standard_normal(m)


def test_zero_perturbations():
    w, T = da.etkf(np.zeros((7, 4)), np.ones(7))
    assert np.array_equal(w, np.zeros(4))
    assert np.allclose(T, np.eye(4), atol=0, rtol=0) or np.abs(T - np.eye(4)).max() < 1e-15


def test_one_member_closed_form():
    y = np.array([[0.5], [-1.5], [2.0]])
    d = np.array([1.0, 2.0, -0.5])
    w, T = da.etkf(y, d)
    yy = float((y[:, 0] ** 2).sum())
    assert abs(w[0] - float(y[:, 0] @ d) / (1 + yy)) < 1e-15
    assert abs(T[0, 0] - 1 / np.sqrt(1 + yy)) < 1e-15


def test_defining_identity_and_woodbury():
    for (m, n, seed) in ((50, 20, 1), (20, 50, 2), (128, 128, 3)):
        Y, d = _case(m, n, seed)
        w, T = da.etkf(Y, d)
        A = np.eye(n) + Y.T @ Y
        assert np.abs(T - T.T).max() < 1e-13
        assert np.abs(T @ A @ T - np.eye(n)).max() < 1e-12
        # Woodbury: A^{-1} Y^T d = Y^T (I_m + Y Y^T)^{-1} d ; A^{-1} = I - Y^T (I_m + Y Y^T)^{-1} Y = T^2
        w2 = Y.T @ np.linalg.solve(np.eye(m) + Y @ Y.T, d)
        assert np.abs(w - w2).max() < 1e-12 * max(1.0, np.abs(w).max())
        T2 = np.eye(n) - Y.T @ np.linalg.solve(np.eye(m) + Y @ Y.T, Y)
        assert np.abs(T @ T - T2).max() < 1e-12
