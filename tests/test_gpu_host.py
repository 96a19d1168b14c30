"""wcsvd_batched_host (the end-to-end entry point with host buffers; include/wcsvd.h): chunked
H2D / kernel / D2H pipeline inside one call. Its outputs must be bitwise those of the device-pointer
entry point on the same inputs (per-matrix determinism), for pinned and pageable, uniform and
mixed-size batches, full and values-only."""
import numpy as np
import pytest
import torch

import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc

pytestmark = pytest.mark.gpu


def _dev(A):
    S, U, V, info = wc.svd_batched(A.cuda(), return_info=True)
    torch.cuda.synchronize()
    return S.cpu(), U.cpu(), V.cpu(), info.cpu().numpy()


@pytest.mark.parametrize("pinned", [True, False])
def test_host_uniform_bitwise_equals_device(pinned):
    mats = workloads.get_config("C2", batch=1500).matrices()
    A = torch.from_numpy(np.stack(mats))
    if pinned:
        A = A.pin_memory()
    S, U, V, info = wc.svd_batched_host(A, return_info=True)
    Sd, Ud, Vd, infod = _dev(A)
    assert torch.equal(S, Sd) and torch.equal(U, Ud) and torch.equal(V, Vd)
    assert np.array_equal(info, infod) and (info > 0).all()


def test_host_mixed_list_bitwise_equals_device():
    cfg = workloads.get_config("C5", batch=40)
    mats = [torch.from_numpy(a).pin_memory() for a in cfg.matrices()]
    S, U, V, info = wc.svd_batched_host(mats, return_info=True)
    Sd, Ud, Vd, infod = wc.svd_batched([a.cuda() for a in mats], return_info=True)
    torch.cuda.synchronize()
    for k in range(len(mats)):
        assert torch.equal(S[k], Sd[k].cpu()) and torch.equal(U[k], Ud[k].cpu()) and torch.equal(V[k], Vd[k].cpu()), k
    assert np.array_equal(info, infod.cpu().numpy())


def test_host_values_only_and_preallocated_out():
    mats = workloads.get_config("C3", batch=20).matrices()
    A = torch.from_numpy(np.stack(mats)).pin_memory()
    S0, _, _ = wc.svd_batched_host(A, compute_uv=False)
    out = wc.svd_batched_host(A)
    S1, U1, V1 = wc.svd_batched_host(A, out=(out[0], out[1].transpose(1, 2), out[2].transpose(1, 2)))
    assert torch.equal(S0, S1)
    Sd, Ud, Vd, _ = _dev(A)
    assert torch.equal(S1, Sd) and torch.equal(U1, Ud) and torch.equal(V1, Vd)
