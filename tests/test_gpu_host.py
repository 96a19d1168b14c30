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


def test_host_mixed_chunked_bitwise_equals_device():
    # >= 300 mixed-size matrices take the chunked path (3 equal-cost chunks, three staging sets)
    rng = np.random.default_rng(77)
    shapes = [(int(rng.integers(8, 97)), int(rng.integers(8, 97))) for _ in range(320)]
    mats = [torch.from_numpy(workloads.gaussian(workloads.matrix_rng(900, k), m, n)).pin_memory()
            for k, (m, n) in enumerate(shapes)]
    S, U, V, info = wc.svd_batched_host(mats, return_info=True)
    Sd, Ud, Vd, infod = wc.svd_batched([a.cuda() for a in mats], return_info=True)
    torch.cuda.synchronize()
    for k in range(len(mats)):
        assert torch.equal(S[k], Sd[k].cpu()) and torch.equal(U[k], Ud[k].cpu()) and torch.equal(V[k], Vd[k].cpu()), k
    assert np.array_equal(info, infod.cpu().numpy()) and (info > 0).all()


@pytest.mark.parametrize("route", ["1", "0"])
def test_host_zero_copy_and_staged_routes_bitwise_equal_device(route, monkeypatch):
    # the zero-copy route (every host buffer mapped: kernels read A / write S, U, V in host memory) and
    # the staged pipeline must both return the device entry point's bits; pageable outputs make the
    # zero-copy route fall back to the pipeline
    monkeypatch.setenv("WCSVD_HOST_ZEROCOPY", route)
    shapes = [(130, 100), (100, 150), (256, 256), (64, 64), (300, 170), (40, 24), (1024, 96), (97, 301)]
    mats = [torch.from_numpy(workloads.gaussian(workloads.matrix_rng(910, k), m, n)).pin_memory()
            for k, (m, n) in enumerate(shapes)]
    Sd, Ud, Vd, infod = wc.svd_batched([a.cuda() for a in mats], return_info=True)
    torch.cuda.synchronize()
    for pinned_out in (True, False):
        ks = [min(m, n) for (m, n) in shapes]
        out = ([torch.empty(k, dtype=torch.float64, pin_memory=pinned_out) for k in ks],
               [torch.empty(k, m, dtype=torch.float64, pin_memory=pinned_out) for k, (m, _) in zip(ks, shapes)],
               [torch.empty(k, n, dtype=torch.float64, pin_memory=pinned_out) for k, (_, n) in zip(ks, shapes)])
        S, U, V, info = wc.svd_batched_host(mats, return_info=True, out=out)
        for k in range(len(mats)):
            assert torch.equal(S[k], Sd[k].cpu()) and torch.equal(U[k], Ud[k].cpu()) and torch.equal(V[k], Vd[k].cpu()), k
        assert np.array_equal(info, infod.cpu().numpy()) and (info > 0).all()


def test_host_values_only_and_preallocated_out():
    mats = workloads.get_config("C3", batch=20).matrices()
    A = torch.from_numpy(np.stack(mats)).pin_memory()
    S0, _, _ = wc.svd_batched_host(A, compute_uv=False)
    out = wc.svd_batched_host(A)
    S1, U1, V1 = wc.svd_batched_host(A, out=(out[0], out[1].transpose(1, 2), out[2].transpose(1, 2)))
    assert torch.equal(S0, S1)
    Sd, Ud, Vd, _ = _dev(A)
    assert torch.equal(S1, Sd) and torch.equal(U1, Ud) and torch.equal(V1, Vd)


def test_host_strided_ld_and_host_info_through_the_c_abi():
    # column-major host blocks with lda > m and ldu / ldv > m / n (the 2-D copy path), pageable numpy
    # memory, per-matrix host info; compared bitwise with the device entry point.
    import ctypes
    rng = workloads.matrix_rng(880, 0)
    shapes = [(70, 50), (50, 70), (130, 120), (64, 64)]
    L = wc.lib()
    B = len(shapes)
    m = np.array([s[0] for s in shapes], dtype=np.int32)
    n = np.array([s[1] for s in shapes], dtype=np.int32)
    k = np.minimum(m, n)
    lda, ldu, ldv = m + 3, m + 5, n + 2
    A = [np.asfortranarray(np.vstack([rng.standard_normal((mm, nn)), np.zeros((3, nn))])) for mm, nn in shapes]
    S = [np.zeros(kk) for kk in k]
    U = [np.zeros((lu, kk), order="F") for lu, kk in zip(ldu, k)]
    V = [np.zeros((lv, kk), order="F") for lv, kk in zip(ldv, k)]
    ptrs = lambda xs: np.array([x.ctypes.data for x in xs], dtype=np.uint64)
    pa, ps, pu, pv = ptrs(A), ptrs(S), ptrs(U), ptrs(V)
    info = np.zeros(B, dtype=np.int32)
    opts = wc.OptsT()
    opts.struct_size = ctypes.sizeof(wc.OptsT)
    opts.ldu, opts.ldv, opts.info = ldu.ctypes.data, ldv.ctypes.data, info.ctypes.data
    rc = L.wcsvd_batched_host(B, m.ctypes.data, n.ctypes.data, pa.ctypes.data, lda.ctypes.data, ps.ctypes.data,
                              pu.ctypes.data, pv.ctypes.data, 0.0, 0, None, ctypes.byref(opts))
    assert rc == 0 and (info > 0).all()
    for b, (mm, nn) in enumerate(shapes):
        # the device entry point on the same column-major matrix (row-major [n, m] = column-major m x n)
        kk = int(k[b])
        Ad = torch.from_numpy(np.ascontiguousarray(A[b][:mm, :].T)).cuda()
        Sd = torch.empty(kk, dtype=torch.float64, device="cuda")
        Ud = torch.empty(kk, mm, dtype=torch.float64, device="cuda")
        Vd = torch.empty(kk, nn, dtype=torch.float64, device="cuda")
        wc.svd_batched_raw([mm], [nn], [Ad.data_ptr()], [mm], [Sd.data_ptr()], [Ud.data_ptr()], [Vd.data_ptr()],
                           stream=torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        assert np.array_equal(S[b], Sd.cpu().numpy())
        assert np.array_equal(U[b][:mm, :], Ud.cpu().numpy().T) and np.array_equal(V[b][:nn, :], Vd.cpu().numpy().T)
        assert not U[b][mm:, :].any() and not V[b][nn:, :].any()  # rows past m / n untouched
