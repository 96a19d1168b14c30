"""CPU oracle for the batched one-sided Jacobi SVD -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package. The product package
``paper_conf_sc_xiaopxsmmlzt22_b200`` never imports it; the two share no code.

The arithmetic lives in plain C (``oracle/oracle.c`` + ``oracle_body.inc``): a textbook cyclic
one-sided Jacobi SVD in long double, written from PAPER.md:47-84 (§II.A-C, eq 1-4)
(§IV.B transpose) and PAPER.md:181 (§III.C), with the readings of SURVEY.md §8(c) / DESIGN.md §3.
This module only compiles it, marshals numpy arrays and returns results.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import sys
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")
_SRC = [os.path.join(_HERE, "oracle.c"), os.path.join(_HERE, "oracle_body.inc")]

__all__ = ["build", "svd", "svd_batch", "syevj", "OracleResult", "ldbl_mant_dig"]


def build(force: bool = False, native: bool = False, out: str | None = None) -> str:
    """Compile the oracle with gcc (plain C, OpenMP over matrices). Returns the .so path.

    ``native=True`` adds ``-march=native`` (used by bench.py for the timing baseline, built into a
    scratch path on the box it runs on); the default build is portable x86-64.
    """
    out = out or _LIB
    if not force and os.path.exists(out):
        if os.path.getmtime(out) >= max(os.path.getmtime(s) for s in _SRC):
            return out
    cmd = ["gcc", "-O3", "-fPIC", "-shared", "-fopenmp", "-ffp-contract=off", "-std=c11"]
    if native:
        cmd.append("-march=native")
    cmd += [_SRC[0], "-o", out + ".tmp", "-lm"]
    subprocess.run(cmd, check=True, cwd=_HERE)
    os.replace(out + ".tmp", out)
    return out


_lib_cache: dict[str, ctypes.CDLL] = {}


def _lib(path: str | None = None) -> ctypes.CDLL:
    path = path or build()
    if path in _lib_cache:
        return _lib_cache[path]
    lib = ctypes.CDLL(path)
    P = ctypes.c_void_p
    I = ctypes.c_int
    D = ctypes.c_double
    for sfx in ("ld", "d"):
        f = getattr(lib, f"oracle_svd_{sfx}")
        f.argtypes = [I, I, P, I, D, I, P, P, P, P, P]
        f.restype = I
        g = getattr(lib, f"oracle_svd_batch_{sfx}")
        g.argtypes = [I, P, P, P, P, D, I, P, P, P, P, P]
        g.restype = None
    lib.oracle_syevj_ld.argtypes = [I, P, D, I, P, P]
    lib.oracle_syevj_ld.restype = I
    lib.oracle_ldbl_mant_dig.restype = I
    lib.oracle_set_threads.argtypes = [I]
    lib.oracle_set_threads.restype = None
    lib.oracle_get_threads.restype = I
    _lib_cache[path] = lib
    return lib


def ldbl_mant_dig() -> int:
    return _lib().oracle_ldbl_mant_dig()


def threads_in_effect(lib_path: str | None = None) -> int:
    return _lib(lib_path).oracle_get_threads()


@dataclass
class OracleResult:
    S: np.ndarray  # (k,)
    U: np.ndarray  # (m, k)
    V: np.ndarray  # (n, k)
    sweeps: int
    rotations: int
    converged: bool


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def svd(A: np.ndarray, tol: float = 0.0, max_sweeps: int = 0, precision: str = "ld") -> OracleResult:
    """Economy SVD of one real matrix A (m x n) by the oracle. ``precision`` 'ld' (parity) or 'd'."""
    A = np.asarray(A, dtype=np.float64)
    m, n = A.shape
    k = min(m, n)
    Af = np.asfortranarray(A)
    S = np.zeros(k)
    U = np.zeros((m, k), order="F")
    V = np.zeros((n, k), order="F")
    sw = ctypes.c_int(0)
    rot = ctypes.c_longlong(0)
    fn = getattr(_lib(), f"oracle_svd_{precision}")
    rc = fn(m, n, _ptr(Af), m, float(tol), int(max_sweeps), _ptr(S), _ptr(U), _ptr(V),
            ctypes.addressof(sw), ctypes.addressof(rot))
    if rc == -2:
        raise MemoryError("oracle allocation failed")
    return OracleResult(S, np.ascontiguousarray(U), np.ascontiguousarray(V), sw.value, rot.value, rc == 0)


def svd_batch(As: list[np.ndarray], tol: float = 0.0, max_sweeps: int = 0, precision: str = "ld",
              threads: int | None = None, lib_path: str | None = None):
    """Batched oracle (OpenMP over matrices, largest first). Returns (S list, U list, V list, info)."""
    lib = _lib(lib_path)
    B = len(As)
    Afs = [np.asfortranarray(np.asarray(a, dtype=np.float64)) for a in As]
    ms = np.array([a.shape[0] for a in Afs], dtype=np.int32)
    ns = np.array([a.shape[1] for a in Afs], dtype=np.int32)
    ks = np.minimum(ms, ns)
    Ss = [np.zeros(k) for k in ks]
    Us = [np.zeros((m, k), order="F") for m, k in zip(ms, ks)]
    Vs = [np.zeros((n, k), order="F") for n, k in zip(ns, ks)]
    info = np.zeros(B, dtype=np.int32)
    cost = ks.astype(np.float64) ** 2 * np.maximum(ms, ns)
    order = np.argsort(-cost, kind="stable").astype(np.int32)
    arr = lambda lst: (ctypes.c_void_p * B)(*[_ptr(x) for x in lst])
    if threads is not None:
        lib.oracle_set_threads(int(threads))
    fn = getattr(lib, f"oracle_svd_batch_{precision}")
    fn(B, _ptr(ms), _ptr(ns), arr(Afs), _ptr(ms), float(tol), int(max_sweeps), arr(Ss), arr(Us), arr(Vs),
       _ptr(info), _ptr(order))
    return Ss, [np.ascontiguousarray(u) for u in Us], [np.ascontiguousarray(v) for v in Vs], info


def syevj(B: np.ndarray, tol: float = 0.0, max_sweeps: int = 0):
    """Two-sided cyclic Jacobi EVD. Returns (lambda unsorted, J, sweeps)."""
    B = np.asfortranarray(np.asarray(B, dtype=np.float64))
    n = B.shape[0]
    lam = np.zeros(n)
    J = np.zeros((n, n), order="F")
    sw = _lib().oracle_syevj_ld(n, _ptr(B), float(tol), int(max_sweeps), _ptr(lam), _ptr(J))
    return lam, np.ascontiguousarray(J), sw


if __name__ == "__main__":  # pragma: no cover
    print(build(force="--force" in sys.argv))
