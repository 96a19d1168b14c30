"""B200-native batched one-sided Jacobi SVD (the W-cycle SVD hot path, Xiao et al., SC'22).

Thin Python binding over the C-ABI in ``include/wcsvd.h`` (``libwcsvd.so``, CUDA sm_100a).
This module only marshals arguments: every numerical step runs in the library's CUDA kernels.
PyTorch provides device memory and the current stream. There is no CPU fallback: if the library
or a CUDA device is missing, calls raise.

Layout: torch tensors are row-major, the C-ABI is column-major. A contiguous m x n tensor is the
column-major n x m matrix A^T (lda = n); we factor that and swap the roles of U and V, which costs
no copies (U and V are returned as transposed views of contiguous buffers).
"""
from __future__ import annotations

import ctypes
import os
from typing import Sequence

import numpy as np

__all__ = ["svd_batched", "svd_batched_host", "etkf_analysis", "svd_batched_raw", "plan", "round_robin", "lib", "WcsvdError",
           "PATH_L0", "PATH_GRAM", "PATH_WCYCLE", "PATH_PANEL", "L0_TWO_PHASE_VARIANTS", "library_path"]

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.environ.get("WCSVD_LIBRARY") or os.path.join(_HERE, "libwcsvd.so")  # env: experiment builds

PATH_AUTO, PATH_L0, PATH_GRAM, PATH_WCYCLE, PATH_PANEL = 0, 1, 2, 3, 4
# Level-0 kernel variants that run the two-phase kernel (csrc/kernels.h kTP32, kTP64; csrc/l0_tp.cu)
L0_TWO_PHASE_VARIANTS = (7, 8)
WCSVD_OK, WCSVD_ENOTSUP, WCSVD_ECUDA, WCSVD_ENOMEM = 0, -100, -101, -102


class WcsvdError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"wcsvd error {code}: {msg}")
        self.code = code


class PlanT(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int), ("n", ctypes.c_int), ("M", ctypes.c_int), ("N", ctypes.c_int),
                ("swapped", ctypes.c_int), ("path", ctypes.c_int), ("n_pad", ctypes.c_int),
                ("m_pad", ctypes.c_int), ("w", ctypes.c_int), ("w2", ctypes.c_int),
                ("variant", ctypes.c_int), ("cost", ctypes.c_double)]


class OptsT(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_size_t), ("ldu", ctypes.c_void_p), ("ldv", ctypes.c_void_p),
                ("info", ctypes.c_void_p), ("sweeps_inner", ctypes.c_void_p),
                ("workspace", ctypes.c_void_p), ("workspace_bytes", ctypes.c_size_t),
                ("force_path", ctypes.c_int), ("force_w", ctypes.c_int), ("wcycle_sweeps", ctypes.c_int),
                ("inner_sweeps", ctypes.c_int), ("pair_warps", ctypes.c_int), ("cluster_ctas", ctypes.c_int),
                ("f32_compute", ctypes.c_int)]


_lib = None


def library_path() -> str:
    return _LIB_PATH


def lib() -> ctypes.CDLL:
    """Load libwcsvd.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise WcsvdError(-101, f"{_LIB_PATH} not built; run __graft_entry__.build() "
                               "(or python paper_conf_sc_xiaopxsmmlzt22_b200/build.py)")
    L = ctypes.CDLL(_LIB_PATH)
    P, I, D = ctypes.c_void_p, ctypes.c_int, ctypes.c_double
    L.wcsvd_batched.argtypes = [I, P, P, P, P, P, P, P, D, I, P]
    L.wcsvd_batched.restype = I
    L.wcsvd_batched_ex.argtypes = [I, P, P, P, P, P, P, P, D, I, P, ctypes.POINTER(OptsT)]
    L.wcsvd_batched_ex.restype = I
    L.wcsvd_batched_f32_ex.argtypes = [I, P, P, P, P, P, P, P, ctypes.c_float, I, P, ctypes.POINTER(OptsT)]
    L.wcsvd_batched_f32_ex.restype = I
    L.wcsvd_batched_host.argtypes = [I, P, P, P, P, P, P, P, D, I, P, ctypes.POINTER(OptsT)]
    L.wcsvd_batched_host.restype = I
    L.wcsvd_workspace_size.argtypes = [I, P, P]
    L.wcsvd_workspace_size.restype = ctypes.c_size_t
    L.wcsvd_status_string.argtypes = [I]
    L.wcsvd_status_string.restype = ctypes.c_char_p
    L.wcsvd_plan.argtypes = [I, I, I, I, ctypes.POINTER(PlanT)]
    L.wcsvd_plan.restype = I
    L.wcsvd_round_robin.argtypes = [I, I, P]
    L.wcsvd_round_robin.restype = I
    L.wcsvd_version.restype = ctypes.c_char_p
    L.wcsvd_etkf_analysis.argtypes = [I, P, P, P, P, P, P, P, P, P]
    L.wcsvd_etkf_analysis.restype = I
    L.wcsvd_trim_workspace.argtypes = []
    L.wcsvd_trim_workspace.restype = I
    _lib = L
    return L


def _check(code: int):
    if code != WCSVD_OK:
        raise WcsvdError(code, lib().wcsvd_status_string(code).decode())


def plan(m: int, n: int, force_path: int = 0, force_w: int = 0) -> dict:
    """Planner introspection (host-only): the per-matrix plan as a dict."""
    p = PlanT()
    _check(lib().wcsvd_plan(int(m), int(n), int(force_path), int(force_w), ctypes.byref(p)))
    return {f: getattr(p, f) for f, _ in PlanT._fields_}


def round_robin(np_: int, step: int) -> list:
    """The round-robin pairs (i, j) of `step` for `np_` indices (host-only)."""
    buf = (ctypes.c_int * np_)()
    if lib().wcsvd_round_robin(int(np_), int(step), buf) != 0:
        raise ValueError("bad round-robin arguments")
    return [(buf[2 * k], buf[2 * k + 1]) for k in range(np_ // 2)]


def _check_out(t, shape, dtype, cuda: bool, name: str):
    """A caller-supplied output buffer must match exactly (the C-ABI writes through raw pointers)."""
    if t is None:
        return
    if tuple(t.shape) != tuple(shape) or t.dtype != dtype or not t.is_contiguous() or bool(t.is_cuda) != cuda:
        where = "CUDA" if cuda else "host"
        raise ValueError(f"out buffer {name}: expected a contiguous {where} {dtype} tensor of shape "
                         f"{tuple(shape)}, got {tuple(t.shape)} {t.dtype} contiguous={t.is_contiguous()} "
                         f"cuda={t.is_cuda}")


def _arr_i32(x) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(x, dtype=np.int32))


def _arr_ptr(x) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(x, dtype=np.uint64))


def svd_batched_raw(m, n, A_ptrs, lda, S_ptrs, U_ptrs=None, V_ptrs=None, tol: float = 0.0,
                    max_sweeps: int = 0, stream: int = 0, ldu=None, ldv=None, info_ptr: int = 0,
                    sweeps_inner_ptr: int = 0, workspace_ptr: int = 0, workspace_bytes: int = 0,
                    force_path: int = 0, force_w: int = 0, wcycle_sweeps: int = 0,
                    inner_sweeps: int = 0, pair_warps: int = 0, cluster_ctas: int = 0, f32_compute: int = 0,
                    fp32: bool = False) -> None:
    """Direct C-ABI call with column-major device pointers (integers). Raises WcsvdError.
    fp32=True calls wcsvd_batched_f32_ex (float data)."""
    m, n, lda = _arr_i32(m), _arr_i32(n), _arr_i32(lda)
    B = len(m)
    Ap, Sp = _arr_ptr(A_ptrs), _arr_ptr(S_ptrs)
    Up = _arr_ptr(U_ptrs) if U_ptrs is not None else None
    Vp = _arr_ptr(V_ptrs) if V_ptrs is not None else None
    keep = []
    opts = OptsT()
    opts.struct_size = ctypes.sizeof(OptsT)
    if ldu is not None:
        a = _arr_i32(ldu); keep.append(a); opts.ldu = a.ctypes.data
    if ldv is not None:
        a = _arr_i32(ldv); keep.append(a); opts.ldv = a.ctypes.data
    opts.info = info_ptr or None
    opts.sweeps_inner = sweeps_inner_ptr or None
    opts.workspace = workspace_ptr or None
    opts.workspace_bytes = workspace_bytes
    opts.force_path, opts.force_w, opts.wcycle_sweeps, opts.inner_sweeps = force_path, force_w, wcycle_sweeps, inner_sweeps
    opts.pair_warps = pair_warps
    opts.cluster_ctas = cluster_ctas
    opts.f32_compute = f32_compute
    fn = lib().wcsvd_batched_f32_ex if fp32 else lib().wcsvd_batched_ex
    rc = fn(B, m.ctypes.data, n.ctypes.data, Ap.ctypes.data, lda.ctypes.data,
            Sp.ctypes.data, Up.ctypes.data if Up is not None else None,
            Vp.ctypes.data if Vp is not None else None, float(tol), int(max_sweeps),
            stream or None, ctypes.byref(opts))
    _check(rc)


def svd_batched(A, tol: float = 0.0, max_sweeps: int = 0, compute_uv: bool = True,
                return_info: bool = False, out=None, compute_u: bool | None = None,
                compute_v: bool | None = None, **kw):
    """Batched economy SVD of fp64 (or fp32: wcsvd_batched_f32) CUDA tensors on the current stream.

    A: tensor [B, m, n] (contiguous) or a sequence of 2-D tensors (sizes may differ).
    Returns (S, U, V) with A = U diag(S) V^T; for a batched tensor S [B, k], U [B, m, k],
    V [B, n, k] (U, V are transposed views); for a list, lists of tensors. With return_info,
    also the per-matrix int32 info tensor (sweeps, -1 not converged, -2 non-finite).
    ``out`` = (S, Ubuf, Vbuf) preallocated as returned by a previous call (batched form only).
    ``compute_u`` / ``compute_v`` (default: ``compute_uv``) select the factors; an unrequested factor
    is returned as None and, when it is the square one, is not accumulated at all (values / U-only
    mode; vector signs then follow the returned factor).
    """
    import torch

    cu = compute_uv if compute_u is None else compute_u
    cv = compute_uv if compute_v is None else compute_v

    if not torch.cuda.is_available():
        raise WcsvdError(WCSVD_ECUDA, "no CUDA device (this library has no CPU fallback)")
    stream = torch.cuda.current_stream().cuda_stream
    if isinstance(A, torch.Tensor):
        if A.dim() != 3 or A.dtype not in (torch.float64, torch.float32) or not A.is_cuda:
            raise ValueError("A must be a float64 or float32 CUDA tensor [B, m, n]")
        A = A.contiguous()
        B, m, n = A.shape
        k = min(m, n)
        dev = A.device
        dt = A.dtype
        es = A.element_size()
        if out is not None:
            S, Ubuf, Vbuf = out
            _check_out(S, (B, k), dt, True, "S")
            _check_out(Ubuf, (B, k, m), dt, True, "U")
            _check_out(Vbuf, (B, k, n), dt, True, "V")
            for t in (S, Ubuf, Vbuf):
                if t is not None and t.device != dev:
                    raise ValueError("out buffers must be on the device of A")
        else:
            S = torch.empty(B, k, dtype=dt, device=dev)
            Ubuf = torch.empty(B, k, m, dtype=dt, device=dev) if cu else None
            Vbuf = torch.empty(B, k, n, dtype=dt, device=dev) if cv else None
        info = torch.empty(B, dtype=torch.int32, device=dev) if return_info else None
        idx = np.arange(B, dtype=np.uint64)
        a_ptr = A.data_ptr() + idx * np.uint64(es * m * n)
        s_ptr = S.data_ptr() + idx * np.uint64(es * k)
        # column-major view: the library factors A^T (n x m, lda = n); its "U" (n x k) is our V,
        # its "V" (m x k) is our U.
        u_ptr = (Vbuf.data_ptr() + idx * np.uint64(es * k * n)) if Vbuf is not None else None
        v_ptr = (Ubuf.data_ptr() + idx * np.uint64(es * k * m)) if Ubuf is not None else None
        svd_batched_raw(np.full(B, n), np.full(B, m), a_ptr, np.full(B, n), s_ptr, u_ptr, v_ptr,
                        tol=tol, max_sweeps=max_sweeps, stream=stream,
                        info_ptr=info.data_ptr() if info is not None else 0, fp32=(es == 4), **kw)
        U = Ubuf.transpose(1, 2) if Ubuf is not None else None
        V = Vbuf.transpose(1, 2) if Vbuf is not None else None
        return (S, U, V, info) if return_info else (S, U, V)
    # list of 2-D tensors
    As = [a.contiguous() for a in A]
    for a in As:
        if a.dim() != 2 or a.dtype not in (torch.float64, torch.float32) or not a.is_cuda:
            raise ValueError("each matrix must be a 2-D float64 or float32 CUDA tensor")
    if len({a.dtype for a in As}) > 1:
        raise ValueError("all matrices of a batch must share one dtype")
    B = len(As)
    if B == 0:
        return ([], [], []) if not return_info else ([], [], [], None)
    dev = As[0].device
    dt = As[0].dtype
    ms = [a.shape[0] for a in As]
    ns = [a.shape[1] for a in As]
    ks = [min(x, y) for x, y in zip(ms, ns)]
    Ss = [torch.empty(k, dtype=dt, device=dev) for k in ks]
    Ub = [torch.empty(k, mm, dtype=dt, device=dev) for k, mm in zip(ks, ms)] if cu else None
    Vb = [torch.empty(k, nn, dtype=dt, device=dev) for k, nn in zip(ks, ns)] if cv else None
    info = torch.empty(B, dtype=torch.int32, device=dev) if return_info else None
    svd_batched_raw(ns, ms, [a.data_ptr() for a in As], ns, [s.data_ptr() for s in Ss],
                    [v.data_ptr() for v in Vb] if Vb is not None else None,
                    [u.data_ptr() for u in Ub] if Ub is not None else None,
                    tol=tol, max_sweeps=max_sweeps, stream=stream,
                    info_ptr=info.data_ptr() if info is not None else 0, fp32=(dt == torch.float32), **kw)
    Us = [u.T for u in Ub] if Ub is not None else None
    Vs = [v.T for v in Vb] if Vb is not None else None
    return (Ss, Us, Vs, info) if return_info else (Ss, Us, Vs)


def _host_call(ms, ns, a_ptrs, s_ptrs, u_ptrs, v_ptrs, tol, max_sweeps, info, kw):
    opts = OptsT()
    opts.struct_size = ctypes.sizeof(OptsT)
    opts.info = info.ctypes.data if info is not None else None
    for key in ("force_path", "force_w", "wcycle_sweeps", "inner_sweeps", "pair_warps", "cluster_ctas", "f32_compute"):
        setattr(opts, key, int(kw.pop(key, 0)))
    if kw:
        raise TypeError(f"unexpected arguments {sorted(kw)}")
    import torch
    stream = torch.cuda.current_stream().cuda_stream
    mm, nn = _arr_i32(ms), _arr_i32(ns)
    a_ptr, s_ptr = _arr_ptr(a_ptrs), _arr_ptr(s_ptrs)
    u_ptr = _arr_ptr(u_ptrs) if u_ptrs is not None else None
    v_ptr = _arr_ptr(v_ptrs) if v_ptrs is not None else None
    rc = lib().wcsvd_batched_host(len(mm), mm.ctypes.data, nn.ctypes.data, a_ptr.ctypes.data, mm.ctypes.data,
                                  s_ptr.ctypes.data, u_ptr.ctypes.data if u_ptr is not None else None,
                                  v_ptr.ctypes.data if v_ptr is not None else None, float(tol), int(max_sweeps),
                                  stream or None, ctypes.byref(opts))
    _check(rc)


def svd_batched_host(A, tol: float = 0.0, max_sweeps: int = 0, compute_uv: bool = True,
                     return_info: bool = False, out=None, **kw):
    """End-to-end batched SVD of HOST fp64 data (wcsvd_batched_host): the host -> device copies, the
    iteration and the device -> host copies run inside one library call, pipelined over chunks (the
    copies overlap the kernels). A: host tensor [B, m, n] or a list of host 2-D tensors (sizes may
    differ); pin them (``pin_memory()``) for full overlap. Returns host (S, U, V) shaped like
    ``svd_batched``'s (U, V are transposed views of row-major [k, m] / [k, n] buffers), pinned when A
    is. ``out`` = (S, Ubuf, Vbuf) preallocated host buffers: tensors [B, k], [B, k, m], [B, k, n] (tensor
    form) or lists of [k], [k, m], [k, n] (list form). Synchronous. With return_info, also the per-matrix info as a numpy int32 array.
    """
    import torch

    if not torch.cuda.is_available():
        raise WcsvdError(WCSVD_ECUDA, "no CUDA device (this library has no CPU fallback)")
    info = None
    if isinstance(A, torch.Tensor):
        if A.dim() != 3 or A.dtype != torch.float64 or A.is_cuda:
            raise ValueError("A must be a float64 host tensor [B, m, n]")
        A = A.contiguous()
        B, m, n = A.shape
        k = min(m, n)
        if out is not None:
            S, Ubuf, Vbuf = out
            _check_out(S, (B, k), A.dtype, False, "S")
            _check_out(Ubuf, (B, k, m), A.dtype, False, "U")
            _check_out(Vbuf, (B, k, n), A.dtype, False, "V")
        else:
            pin = A.is_pinned()
            S = torch.empty(B, k, dtype=A.dtype, pin_memory=pin)
            Ubuf = torch.empty(B, k, m, dtype=A.dtype, pin_memory=pin) if compute_uv else None
            Vbuf = torch.empty(B, k, n, dtype=A.dtype, pin_memory=pin) if compute_uv else None
        info = np.zeros(B, dtype=np.int32) if return_info else None
        idx = np.arange(B, dtype=np.uint64)
        es = np.uint64(8)
        # column-major view (as svd_batched): the library factors A^T (n x m, lda = n); its U is our V
        _host_call(np.full(B, n), np.full(B, m), A.data_ptr() + idx * (es * np.uint64(m * n)),
                   S.data_ptr() + idx * (es * np.uint64(k)),
                   (Vbuf.data_ptr() + idx * (es * np.uint64(k * n))) if Vbuf is not None else None,
                   (Ubuf.data_ptr() + idx * (es * np.uint64(k * m))) if Ubuf is not None else None,
                   tol, max_sweeps, info, kw)
        U = Ubuf.transpose(1, 2) if Ubuf is not None else None
        V = Vbuf.transpose(1, 2) if Vbuf is not None else None
        return (S, U, V, info) if return_info else (S, U, V)
    As = [a.contiguous() for a in A]
    for a in As:
        if a.dim() != 2 or a.dtype != torch.float64 or a.is_cuda:
            raise ValueError("each matrix must be a 2-D float64 host tensor")
    B = len(As)
    if B == 0:
        return ([], [], []) if not return_info else ([], [], [], None)
    pin = all(a.is_pinned() for a in As)
    ms = [a.shape[0] for a in As]
    ns = [a.shape[1] for a in As]
    ks = [min(x, y) for x, y in zip(ms, ns)]
    if out is not None:  # lists (S, Ubuf, Vbuf) of host buffers [k], [k, m], [k, n]
        Ss, Ub, Vb = out
        if len(Ss) != B or (Ub is not None and len(Ub) != B) or (Vb is not None and len(Vb) != B):
            raise ValueError("out lists must have one buffer per matrix")
        for i in range(B):
            _check_out(Ss[i], (ks[i],), torch.float64, False, f"S[{i}]")
            _check_out(Ub[i] if Ub is not None else None, (ks[i], ms[i]), torch.float64, False, f"U[{i}]")
            _check_out(Vb[i] if Vb is not None else None, (ks[i], ns[i]), torch.float64, False, f"V[{i}]")
    else:
        Ss = [torch.empty(k, dtype=torch.float64, pin_memory=pin) for k in ks]
        Ub = [torch.empty(k, mm, dtype=torch.float64, pin_memory=pin) for k, mm in zip(ks, ms)] if compute_uv else None
        Vb = [torch.empty(k, nn, dtype=torch.float64, pin_memory=pin) for k, nn in zip(ks, ns)] if compute_uv else None
    info = np.zeros(B, dtype=np.int32) if return_info else None
    _host_call(ns, ms, [a.data_ptr() for a in As], [s.data_ptr() for s in Ss],
               [v.data_ptr() for v in Vb] if Vb is not None else None,
               [u.data_ptr() for u in Ub] if Ub is not None else None, tol, max_sweeps, info, kw)
    Us = [u.T for u in Ub] if Ub is not None else None
    Vs = [v.T for v in Vb] if Vb is not None else None
    return (Ss, Us, Vs, info) if return_info else (Ss, Us, Vs)


def etkf_analysis(S, U, V, d):
    """Data-assimilation consumer (wcsvd_etkf_analysis): for each grid
    point with scaled ensemble perturbations Y = U diag(S) V^T (svd_batched's outputs) and scaled
    innovation d, returns (wbar, T) with wbar = (I + Y^T Y)^-1 Y^T d and T = (I + Y^T Y)^-1/2.

    Batched form: S [B, k], U [B, m, k], V [B, n, k] exactly as svd_batched returns them (U, V are
    transposed views of contiguous buffers), d [B, m] -> wbar [B, n], T [B, n, n]. List form: lists of
    the per-matrix tensors -> lists. fp64 CUDA tensors; runs on the current stream."""
    import torch

    if not torch.cuda.is_available():
        raise WcsvdError(WCSVD_ECUDA, "no CUDA device (this library has no CPU fallback)")
    stream = torch.cuda.current_stream().cuda_stream
    batched = isinstance(S, torch.Tensor)
    Ss = list(S) if batched else list(S)
    Us = list(U) if batched else list(U)
    Vs = list(V) if batched else list(V)
    ds = list(d) if batched else list(d)
    B = len(Ss)
    if not (len(Us) == len(Vs) == len(ds) == B):
        raise ValueError("S, U, V, d must have one entry per matrix")
    if B == 0:
        return ([], []) if not batched else (None, None)
    ms, ns, ptrs = [], [], {"S": [], "U": [], "V": [], "d": []}
    keep = []
    for s, u, v, dd in zip(Ss, Us, Vs, ds):
        for t in (s, u, v, dd):
            if t.dtype != torch.float64 or not t.is_cuda:
                raise ValueError("S, U, V, d must be float64 CUDA tensors")
        m, k = u.shape
        n = v.shape[0]
        if v.shape[1] != k or s.numel() != k or k != min(m, n) or dd.numel() != m:
            raise ValueError("shapes must be S [k], U [m, k], V [n, k], d [m] with k = min(m, n)")
        uc, vc = u.t().contiguous(), v.t().contiguous()  # column-major m x k / n x k (no copy for views)
        sc, dc = s.contiguous(), dd.contiguous()
        keep += [uc, vc, sc, dc]
        ms.append(m)
        ns.append(n)
        ptrs["S"].append(sc.data_ptr())
        ptrs["U"].append(uc.data_ptr())
        ptrs["V"].append(vc.data_ptr())
        ptrs["d"].append(dc.data_ptr())
    dev = Ss[0].device
    wb = [torch.empty(n, dtype=torch.float64, device=dev) for n in ns]
    Tb = [torch.empty(n, n, dtype=torch.float64, device=dev) for n in ns]  # written column-major
    mm, nn = _arr_i32(ms), _arr_i32(ns)
    arr = {k: _arr_ptr(v) for k, v in ptrs.items()}
    pw = _arr_ptr([w.data_ptr() for w in wb])
    pt = _arr_ptr([t.data_ptr() for t in Tb])
    _check(lib().wcsvd_etkf_analysis(B, mm.ctypes.data, nn.ctypes.data, arr["S"].ctypes.data, arr["U"].ctypes.data,
                                     arr["V"].ctypes.data, arr["d"].ctypes.data, pw.ctypes.data, pt.ctypes.data,
                                     stream or None))
    Ts = [t.t() for t in Tb]
    if batched:
        return torch.stack(wb), torch.stack(Ts)
    return wb, Ts
