"""Helpers for the -m gpu parity tests: run the CUDA path through the C-ABI binding and compare
with the long-double oracle on the same seeded inputs (oracle/compare.py bars)."""
from __future__ import annotations

import numpy as np

import oracle
from oracle import compare


def gpu_svd_list(mats, **kw):
    """CUDA path on a list of numpy matrices -> lists of numpy (S, U, V) and info."""
    import torch
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc

    dev = torch.device("cuda:0")
    As = [torch.from_numpy(np.ascontiguousarray(a)).to(dev) for a in mats]
    S, U, V, info = wc.svd_batched(As, return_info=True, **kw)
    torch.cuda.synchronize()
    return ([s.cpu().numpy() for s in S], [u.cpu().numpy() for u in U], [v.cpu().numpy() for v in V],
            info.cpu().numpy())


def gpu_svd_tensor(stack: np.ndarray, **kw):
    import torch
    import paper_conf_sc_xiaopxsmmlzt22_b200 as wc

    A = torch.from_numpy(np.ascontiguousarray(stack)).cuda()
    S, U, V, info = wc.svd_batched(A, return_info=True, **kw)
    torch.cuda.synchronize()
    return S.cpu().numpy(), U.cpu().numpy(), V.cpu().numpy(), info.cpu().numpy()


def check_parity(mats, S, U, V, info=None, idx=None, oracle_out=None, bars=None):
    """Compare GPU outputs for mats[i] with the oracle; returns list of Parity; asserts bars."""
    bars = bars or {}
    idx = range(len(mats)) if idx is None else idx
    mats_sel = [mats[i] for i in idx]
    if oracle_out is None:
        So, Uo, Vo, info_o = oracle.svd_batch(mats_sel)
    else:
        So, Uo, Vo, info_o = oracle_out
    res = []
    for j, i in enumerate(idx):
        p = compare.compare(mats[i], S[i], U[i], V[i], So[j], Uo[j], Vo[j])
        res.append(p)
        assert p.ok(**bars), f"matrix {i} shape {mats[i].shape}: {p.as_dict()} info={None if info is None else info[i]} oracle_sweeps={info_o[j]}"
        if info is not None:
            assert info[i] > 0, f"matrix {i} did not converge: info={info[i]}"
    return res
