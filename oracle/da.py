"""CPU oracle of the data-assimilation consumer -- TEST INFRASTRUCTURE ONLY.

Reading R-DA: the paper's application (§V.F) performs one SVD per grid
point of an ensemble data-assimilation system (its refs [36]-[38], are ensemble
Kalman filters); it does not write the analysis out. The oracle is the ensemble transform Kalman
filter's ensemble-space analysis written from its plain definition, in float64, from the scaled
observation-space perturbations Y (m x n) and the scaled innovation d (m) -- NOT from an SVD:

    A    = I_n + Y^T Y                     (the inverse analysis covariance in ensemble space)
    wbar = A^{-1} Y^T d                    (numpy.linalg.solve)
    T    = A^{-1/2}                        (symmetric square root through numpy.linalg.eigh of A)

so the CUDA path (SVD -> wcsvd_etkf_analysis) is checked against an independent route.
"""
from __future__ import annotations

import numpy as np

__all__ = ["etkf"]


def etkf(Y: np.ndarray, d: np.ndarray):
    """(wbar, T) of the ETKF analysis for scaled perturbations Y (m x n) and innovation d (m)."""
    Y = np.asarray(Y, dtype=np.float64)
    d = np.asarray(d, dtype=np.float64)
    n = Y.shape[1]
    A = np.eye(n) + Y.T @ Y
    wbar = np.linalg.solve(A, Y.T @ d)
    lam, Q = np.linalg.eigh(A)
    T = (Q / np.sqrt(lam)) @ Q.T
    return wbar, T
