"""ORACLE — test infrastructure only (see oracle/oracle.c header).

ctypes binding of `oracle/liboracle.so`, a plain C fp64 implementation of every operation
on the hot path, written from the paper as restated in SURVEY.md §8(c).
Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package.  It shares no code with paper_conf_icpp_nelsonrbhhjn15_b200/
(the CUDA product path); the only module both sides use is `synthetic` (seeded inputs).

Functions take and return numpy float64 C-contiguous arrays.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, -O2 -ffp-contract=off, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        d, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        for name in ("oracle_sumfact3d_def", "oracle_sumfact3d"):
            getattr(_lib, name).argtypes = [i64, i32, d, d, d, d, d]
        for name in ("oracle_sumfact2d_def", "oracle_sumfact2d"):
            getattr(_lib, name).argtypes = [i64, i32, d, d, d, d]
        _lib.oracle_local_grad3.argtypes = [i64, i32, d, d, d, d, d]
        _lib.oracle_local_grad3_t.argtypes = [i64, i32, d, d, d, d, d]
        _lib.oracle_ax_e.argtypes = [i64, i32, d, d, d, d]
        for name in ("oracle_ccsdt_d1", "oracle_ccsdt_d2", "oracle_ccsdt_s1"):
            getattr(_lib, name).argtypes = [i32, d, d, d, d]
        _lib.oracle_ccsdt_variant.argtypes = [i32, i32, d]
        _lib.oracle_ccsdt_variant.restype = i32
        _lib.oracle_sumsq.argtypes = [i64, d]
        _lib.oracle_sumsq.restype = ctypes.c_double
        _lib.oracle_energy.argtypes = [d, d, d, d]
        _lib.oracle_energy.restype = ctypes.c_double
    return _lib


def set_threads(n: int) -> None:
    """OpenMP thread count for subsequent oracle calls from this thread (bench.py times
    the oracle on all cores and on one core; no effect on results, which do not depend
    on the thread count)."""
    lib()
    ctypes.CDLL("libgomp.so.1").omp_set_num_threads(int(n))


def _c(a) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.float64)
    return a


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _P1(op) -> int:
    return op.shape[0]


# ---------------------------------------------------------------- spectral family

def sumfact3d(A, B, C, U, level: int = 1) -> np.ndarray:
    """V[e][i][j][k] = sum_lmn A[k][n] B[j][m] C[i][l] U[e][l][m][n]; U shape (N,P1,P1,P1)."""
    A, B, C, U = _c(A), _c(B), _c(C), _c(U)
    P1 = _P1(A)
    assert U.shape[1:] == (P1, P1, P1)
    V = np.empty_like(U)
    fn = lib().oracle_sumfact3d if level == 1 else lib().oracle_sumfact3d_def
    fn(U.shape[0], P1 - 1, _p(A), _p(B), _p(C), _p(U), _p(V))
    return V


def sumfact2d(A, B, U, level: int = 1) -> np.ndarray:
    """V[e][i][j] = sum_lm B[i][l] A[j][m] U[e][l][m]  (V = B U A^T); U shape (N,P1,P1)."""
    A, B, U = _c(A), _c(B), _c(U)
    P1 = _P1(A)
    assert U.shape[1:] == (P1, P1)
    V = np.empty_like(U)
    fn = lib().oracle_sumfact2d if level == 1 else lib().oracle_sumfact2d_def
    fn(U.shape[0], P1 - 1, _p(A), _p(B), _p(U), _p(V))
    return V


def local_grad3(D, U):
    """(ur, us, ut) of Nekbone local_grad3 on U[e][k][j][i]."""
    D, U = _c(D), _c(U)
    P1 = _P1(D)
    ur, us, ut = np.empty_like(U), np.empty_like(U), np.empty_like(U)
    lib().oracle_local_grad3(U.shape[0], P1 - 1, _p(D), _p(U), _p(ur), _p(us), _p(ut))
    return ur, us, ut


def local_grad3_t(D, ur, us, ut):
    D, ur, us, ut = _c(D), _c(ur), _c(us), _c(ut)
    P1 = _P1(D)
    U = np.empty_like(ur)
    lib().oracle_local_grad3_t(ur.shape[0], P1 - 1, _p(D), _p(ur), _p(us), _p(ut), _p(U))
    return U


def ax_e(D, U, G):
    """Nekbone element operator; G shape (N, 6, P1, P1, P1)."""
    D, U, G = _c(D), _c(U), _c(G)
    P1 = _P1(D)
    assert G.shape == (U.shape[0], 6) + U.shape[1:]
    W = np.empty_like(U)
    lib().oracle_ax_e(U.shape[0], P1 - 1, _p(D), _p(U), _p(G), _p(W))
    return W


# ---------------------------------------------------------------- CCSD(T) family
# ext = (h1d, h2d, h3d, p4d, p5d, p6d, kd); arrays are flat, Fortran offsets.

NAMES = ("h1", "h2", "h3", "p4", "p5", "p6", "k")


def _ext(ext) -> np.ndarray:
    e = np.ascontiguousarray(ext, dtype=np.int32)
    assert e.shape == (7,)
    return e


def ccsdt(family: str, variant: int, ext, t3, t2, v2) -> np.ndarray:
    """Return t3 + s_v * contraction (t3 not modified).  family in {'d1','d2','s1'}."""
    e = _ext(ext)
    out = _c(t3).copy()
    fn = {"d1": lib().oracle_ccsdt_d1, "d2": lib().oracle_ccsdt_d2, "s1": lib().oracle_ccsdt_s1}[family]
    t2, v2 = _c(t2), _c(v2)
    fn(int(variant), _p(e), _p(out), _p(t2), _p(v2))
    return out


def ccsdt_fused(family: str, ext, t3, t2s, v2s) -> np.ndarray:
    """Fused form: t3 + sum_{v=1..9, t2s[v-1] is not None} contribution_v,
    applied in ascending v."""
    out = _c(t3).copy()
    for v in range(1, 10):
        if t2s[v - 1] is None:
            continue
        out = ccsdt(family, v, ext, out, t2s[v - 1], v2s[v - 1])
    return out


def variant_table(family: str, variant: int):
    """(storage order as names, sign) for tests."""
    o = np.zeros(6, dtype=np.int32)
    s = lib().oracle_ccsdt_variant({"d1": 1, "d2": 2, "s1": 3}[family], int(variant), _p(o))
    return tuple(NAMES[i] for i in o), int(s)


def sumsq(x) -> float:
    x = _c(x).ravel()
    return float(lib().oracle_sumsq(x.size, _p(x)))


def energy(ext, t3, eps_h, eps_p) -> float:
    e = _ext(ext)
    return float(lib().oracle_energy(_p(e), _p(_c(t3)), _p(_c(eps_h)), _p(_c(eps_p))))


def ccsdt_abs_bound(family: str, ext, t3, t2s, v2s) -> np.ndarray:
    """Componentwise scale for tolerances (R14): |t3| + sum_v |t2_v|.|v2_v| sums,
    i.e. the same contraction evaluated on absolute values with all signs positive."""
    out = np.abs(_c(t3)).copy()
    z = np.zeros_like(out)
    for v in range(1, 10):
        if t2s[v - 1] is None:
            continue
        out += np.abs(ccsdt(family, v, ext, z, np.abs(t2s[v - 1]), np.abs(v2s[v - 1])))
    return out
