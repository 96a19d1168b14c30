"""Data-assimilation consumer on the GPU: batched SVD of the scaled
ensemble perturbations (C4-like 1024 x 128 ensembles, and fewer observations than members) followed
by wcsvd_etkf_analysis, against the independent CPU oracle (oracle/da.py: solve + eigh, no SVD)."""
import numpy as np
import pytest
import torch

import workloads
from oracle import da

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("shape,batch", [((1024, 128), 6), ((100, 128), 4), ((300, 300), 3), ((50, 50), 5)])
def test_etkf_analysis_matches_oracle(shape, batch):
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc

    m, n = shape
    rng = workloads.matrix_rng(4600 + m, n)
    Ys, ds = [], []
    for b in range(batch):
        if shape == (1024, 128):
            Y = workloads.get_config("C4").make(b) * 3.0  # ensemble-like spectrum (kappa 1e4)
        else:
            Y = workloads.gaussian(rng, m, n) / np.sqrt(n - 1)
        Ys.append(Y)
        ds.append(rng.standard_normal(m))
    A = torch.from_numpy(np.stack(Ys)).cuda()
    S, U, V = wc.svd_batched(A)
    d = torch.from_numpy(np.stack(ds)).cuda()
    wbar, T = wc.etkf_analysis(S, U, V, d)
    torch.cuda.synchronize()
    for b in range(batch):
        w_ref, T_ref = da.etkf(Ys[b], ds[b])
        scale_w = max(1.0, np.abs(w_ref).max())
        assert np.abs(wbar[b].cpu().numpy() - w_ref).max() <= 1e-11 * scale_w, b
        assert np.abs(T[b].cpu().numpy() - T_ref).max() <= 1e-11, b
    # list form gives the same bits
    wl, Tl = wc.etkf_analysis(list(S), list(U), list(V), list(d))
    for b in range(batch):
        assert torch.equal(wl[b], wbar[b]) and torch.equal(Tl[b], T[b])
