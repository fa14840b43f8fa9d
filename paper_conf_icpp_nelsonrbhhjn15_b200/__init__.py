"""libbarracuda Python binding: B200-native batched small tensor contractions.

Thin argument marshalling over the C ABI in include/barracuda.h (ctypes): every function
checks dtype / device / contiguity and every tensor's shape or element count against the
sizes it passes (N, p, extents, workspace), then calls the library on the tensors' device
with their `data_ptr()`s and that device's current CUDA stream.  All arithmetic happens in the sm_100a kernels; there is no CPU or
PyTorch fallback (importing raises if libbarracuda.so is missing, and every call raises
BarracudaError on a non-zero status).

Method: Nelson et al., "Generating Efficient Tensor Contractions for GPUs", ICPP 2015
 — see DESIGN.md for the path, the readings of the paper, and the layouts.
"""
from __future__ import annotations

import ctypes
from typing import Optional, Sequence

import torch

from . import _abi
from ._abi import BC_CHECK_WS_DOUBLES, TileDims, lib

__all__ = [
    "BarracudaError", "sumfact3d", "sumfact2d", "local_grad3", "local_grad3_t", "ax_e",
    "ccsdt", "ccsdt_fused", "ccsdt_triples_energy", "check_sumsq", "check_energy", "fill", "launch_count",
    "reset_launch_count", "probe_fp64_tflops", "operand_sizes", "LIB_PATH",
]

LIB_PATH = _abi.LIB_PATH


class BarracudaError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = lib.bc_status_string(status).decode()
        if status == -5:
            msg += f" (cudaError {lib.bc_last_cuda_error()})"
        super().__init__(f"{where}: {msg}")
        self.status = status


def _check(status: int, where: str) -> None:
    if status != 0:
        raise BarracudaError(status, where)


def _stream(t: torch.Tensor) -> ctypes.c_void_p:
    return ctypes.c_void_p(torch.cuda.current_stream(t.device).cuda_stream)


def _dev(t: torch.Tensor, dtype: torch.dtype, name: str, device: Optional[torch.device] = None,
         numel: Optional[int] = None, min_numel: Optional[int] = None) -> int:
    """Validate one tensor argument and return its device pointer: a contiguous CUDA tensor
    of `dtype`, on `device` (when given), with exactly `numel` / at least `min_numel`
    elements (the C ABI takes sizes only through N / p / extents, so a short buffer would
    otherwise become an out-of-bounds device access)."""
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (no CPU path)")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if device is not None and t.device != device:
        raise ValueError(f"{name} is on {t.device}, expected {device}")
    if numel is not None and t.numel() != numel:
        raise ValueError(f"{name} must have {numel} elements, got {t.numel()}")
    if min_numel is not None and t.numel() < min_numel:
        raise ValueError(f"{name} must have >= {min_numel} elements, got {t.numel()}")
    return t.data_ptr()


def _on(dev: torch.device):
    """Context that makes `dev` current for the call (the library launches on the current
    device); CPU tensors are refused here already (there is no CPU path)."""
    if dev.type != "cuda":
        raise ValueError("arguments must be CUDA tensors (no CPU path)")
    return torch.cuda.device(dev)


def _p_of(op: torch.Tensor, name: str) -> int:
    if op.dim() != 2 or op.shape[0] != op.shape[1]:
        raise ValueError(f"{name} must be square (p+1)x(p+1)")
    return op.shape[0] - 1


def _op(op: torch.Tensor, P1: int, dtype, dev, name: str) -> int:
    if tuple(op.shape) != (P1, P1):
        raise ValueError(f"{name} must be {P1}x{P1}, got {tuple(op.shape)}")
    return _dev(op, dtype, name, dev)


def _field(U: torch.Tensor, P1: int, ndim: int, name: str) -> int:
    if U.dim() != ndim + 1 or tuple(U.shape[1:]) != (P1,) * ndim:
        raise ValueError(f"{name} must have shape (N,{','.join(['p+1'] * ndim)}) with p+1={P1}")
    return U.shape[0]


def _out(out: Optional[torch.Tensor], like: torch.Tensor, name: str = "out") -> torch.Tensor:
    if out is None:
        return torch.empty_like(like)
    if tuple(out.shape) != tuple(like.shape):
        raise ValueError(f"{name} must have shape {tuple(like.shape)}, got {tuple(out.shape)}")
    return out


# ----------------------------------------------------------------------------- spectral

def sumfact3d(A, B, C, U, out: Optional[torch.Tensor] = None, check_ws: Optional[torch.Tensor] = None) -> torch.Tensor:
    """V[e][i][j][k] = sum_lmn A[k][n] B[j][m] C[i][l] U[e][l][m][n]  (fp64 or fp32).
    check_ws (fp64, >= 1024 doubles): also leave sum(V^2) in check_ws[0] (fused, fp64 only)."""
    p = _p_of(A, "A")
    P1 = p + 1
    N = _field(U, P1, 3, "U")
    V = _out(out, U)
    dt, dev = U.dtype, U.device
    with _on(dev):
        if check_ws is not None:
            f = torch.float64
            _check(lib.bc_sumfact3d_check(N, p, _op(A, P1, f, dev, "A"), _op(B, P1, f, dev, "B"),
                                          _op(C, P1, f, dev, "C"), _dev(U, f, "U", dev), _dev(V, f, "out", dev),
                                          _dev(check_ws, f, "check_ws", dev, min_numel=BC_CHECK_WS_DOUBLES),
                                          _stream(U)), "bc_sumfact3d_check")
            return V
        fn = {torch.float64: lib.bc_sumfact3d, torch.float32: lib.bc_sumfact3d_f32}.get(dt)
        if fn is None:
            raise TypeError("sumfact3d supports float64 and float32")
        _check(fn(N, p, _op(A, P1, dt, dev, "A"), _op(B, P1, dt, dev, "B"), _op(C, P1, dt, dev, "C"),
                  _dev(U, dt, "U", dev), _dev(V, dt, "out", dev), _stream(U)), "bc_sumfact3d")
    return V


def sumfact2d(A, B, U, out=None) -> torch.Tensor:
    """V[e][i][j] = sum_lm B[i][l] A[j][m] U[e][l][m]  (V = B U A^T)."""
    p = _p_of(A, "A")
    P1 = p + 1
    N = _field(U, P1, 2, "U")
    V = _out(out, U)
    f, dev = torch.float64, U.device
    with _on(dev):
        _check(lib.bc_sumfact2d(N, p, _op(A, P1, f, dev, "A"), _op(B, P1, f, dev, "B"), _dev(U, f, "U", dev),
                                _dev(V, f, "out", dev), _stream(U)), "bc_sumfact2d")
    return V


def local_grad3(D, U, out=None):
    """(ur, us, ut) of Nekbone local_grad3 on U[e][k][j][i]."""
    p = _p_of(D, "D")
    N = _field(U, p + 1, 3, "U")
    if out is None:
        ur, us, ut = (torch.empty_like(U) for _ in range(3))
    else:
        ur, us, ut = (_out(o, U, nm) for o, nm in zip(out, ("ur", "us", "ut")))
    f, dev = torch.float64, U.device
    with _on(dev):
        _check(lib.bc_local_grad3(N, p, _op(D, p + 1, f, dev, "D"), _dev(U, f, "U", dev), _dev(ur, f, "ur", dev),
                                  _dev(us, f, "us", dev), _dev(ut, f, "ut", dev), _stream(U)), "bc_local_grad3")
    return ur, us, ut


def local_grad3_t(D, ur, us, ut, out=None) -> torch.Tensor:
    p = _p_of(D, "D")
    N = _field(ur, p + 1, 3, "ur")
    for t, nm in ((us, "us"), (ut, "ut")):
        _out(t, ur, nm)
    U = _out(out, ur)
    f, dev = torch.float64, ur.device
    with _on(dev):
        _check(lib.bc_local_grad3_t(N, p, _op(D, p + 1, f, dev, "D"), _dev(ur, f, "ur", dev), _dev(us, f, "us", dev),
                                    _dev(ut, f, "ut", dev), _dev(U, f, "out", dev), _stream(ur)), "bc_local_grad3_t")
    return U


def ax_e(D, U, G, out=None) -> torch.Tensor:
    """Nekbone element operator; G has shape (N, 6, p+1, p+1, p+1)."""
    p = _p_of(D, "D")
    N = _field(U, p + 1, 3, "U")
    if tuple(G.shape) != (N, 6) + tuple(U.shape[1:]):
        raise ValueError("G must have shape (N, 6, p+1, p+1, p+1)")
    W = _out(out, U)
    f, dev = torch.float64, U.device
    with _on(dev):
        _check(lib.bc_ax_e(N, p, _op(D, p + 1, f, dev, "D"), _dev(U, f, "U", dev), _dev(G, f, "G", dev),
                           _dev(W, f, "out", dev), _stream(U)), "bc_ax_e")
    return W


# ----------------------------------------------------------------------------- CCSD(T)

def _dims(ext: Sequence[int]) -> TileDims:
    if len(ext) != 7:
        raise ValueError("ext = (h1, h2, h3, p4, p5, p6, k)")
    return TileDims(*[int(x) for x in ext])


def _n3(ext) -> int:
    n = 1
    for x in ext[:6]:
        n *= int(x)
    return n


def operand_sizes(family: str, ext) -> tuple:
    """(numel of the first operand, numel of the second) of one variant: d1 t2[h7,p4,p5,h1],
    v2[h3,h2,p6,h7]; d2 t2[p7,p4,h1,h2], v2[p7,h3,p6,p5]; s1 t1[p4,h1], v2[h3,h2,p6,p5]."""
    h1, h2, h3, p4, p5, p6, k = (int(x) for x in ext)
    return {"d1": (k * p4 * p5 * h1, h3 * h2 * p6 * k), "d2": (k * p4 * h1 * h2, k * h3 * p6 * p5),
            "s1": (p4 * h1, h3 * h2 * p6 * p5)}[family]


def ccsdt(family: str, variant: int, ext, t3: torch.Tensor, t2: torch.Tensor, v2: torch.Tensor) -> torch.Tensor:
    """t3 += s_v * contraction of NWChem sd_t_<family>_<variant> (in place; returns t3).
    family in {'d1','d2','s1'}; ext = (h1,h2,h3,p4,p5,p6,k); flat Fortran-ordered tensors."""
    fn = {"d1": lib.bc_ccsdt_d1, "d2": lib.bc_ccsdt_d2, "s1": lib.bc_ccsdt_s1}[family]
    f, dev = torch.float64, t3.device
    d = _dims(ext)
    na, nb = operand_sizes(family, ext)
    with _on(dev):
        _check(fn(int(variant), ctypes.byref(d), _dev(t3, f, "t3", dev, numel=_n3(ext)),
                  _dev(t2, f, "t2", dev, numel=na), _dev(v2, f, "v2", dev, numel=nb), _stream(t3)),
               f"bc_ccsdt_{family}")
    return t3


def _ptr9(xs, ys, nm, dev, na, nb):
    a, b = _abi.PtrArray9(), _abi.PtrArray9()
    if len(xs) != 9 or len(ys) != 9:
        raise ValueError(f"{nm}: 9 operands per list")
    for v in range(9):
        if xs[v] is not None:
            if ys[v] is None:
                raise ValueError(f"{nm}[{v}]: second operand missing")
            a[v] = _dev(xs[v], torch.float64, f"{nm}[{v}]", dev, numel=na)
            b[v] = _dev(ys[v], torch.float64, f"{nm}v2[{v}]", dev, numel=nb)
    return a, b


def ccsdt_fused(family: str, ext, t3: torch.Tensor, t2s, v2s) -> torch.Tensor:
    """t3 += sum over v with t2s[v-1] not None (in place; returns t3)."""
    fn = {"d1": lib.bc_ccsdt_d1_fused, "d2": lib.bc_ccsdt_d2_fused, "s1": lib.bc_ccsdt_s1_fused}[family]
    dev = t3.device
    a, b = _ptr9(t2s, v2s, "t2", dev, *operand_sizes(family, ext))
    d = _dims(ext)
    with _on(dev):
        _check(fn(ctypes.byref(d), _dev(t3, torch.float64, "t3", dev, numel=_n3(ext)), a, b, _stream(t3)),
               f"bc_ccsdt_{family}_fused")
    return t3


def ccsdt_fused_energy(family: str, ext, t3: torch.Tensor, t2s, v2s, eps_h, eps_p, ws=None) -> torch.Tensor:
    """t3 += the fused family (as ccsdt_fused), then ws[0] = check_energy of the updated t3
    (fused into the tensor-core kernel's store pass where it runs on full cubes).
    Returns ws[0] (device scalar)."""
    fam = {"d1": 1, "d2": 2, "s1": 3}[family]
    dev = t3.device
    f = torch.float64
    if ws is None:
        ws = torch.empty(BC_CHECK_WS_DOUBLES, dtype=f, device=dev)
    a, b = _ptr9(t2s, v2s, "t2", dev, *operand_sizes(family, ext))
    d = _dims(ext)
    h = int(ext[0]) + int(ext[1]) + int(ext[2])
    pp = int(ext[3]) + int(ext[4]) + int(ext[5])
    with _on(dev):
        _check(lib.bc_ccsdt_fused_energy(fam, ctypes.byref(d), _dev(t3, f, "t3", dev, numel=_n3(ext)), a, b,
                                         _dev(eps_h, f, "eps_h", dev, numel=h), _dev(eps_p, f, "eps_p", dev, numel=pp),
                                         _dev(ws, f, "ws", dev, min_numel=BC_CHECK_WS_DOUBLES), _stream(t3)),
               "bc_ccsdt_fused_energy")
    return ws[0]


def ccsdt_triples_energy(ext, s1, d1, d2, eps_h, eps_p, ws=None) -> torch.Tensor:
    """Energy of the t3 built from all (non-None) triples variants, t3 never stored.
    s1 = (t1s, v2s), d1 = (t2s, v2s), d2 = (t2s, v2s): lists of 9 (None = skip).
    Returns ws[0] (device scalar)."""
    f = torch.float64
    dev = eps_h.device
    if ws is None:
        ws = torch.empty(BC_CHECK_WS_DOUBLES, dtype=f, device=dev)
    arrs = []
    for (xs, ys), nm in ((s1, "s1"), (d1, "d1"), (d2, "d2")):
        arrs += list(_ptr9(xs, ys, nm, dev, *operand_sizes(nm, ext)))
    d = _dims(ext)
    h = int(ext[0]) + int(ext[1]) + int(ext[2])
    pp = int(ext[3]) + int(ext[4]) + int(ext[5])
    with _on(dev):
        _check(lib.bc_ccsdt_triples_energy(ctypes.byref(d), *arrs, _dev(eps_h, f, "eps_h", dev, numel=h),
                                           _dev(eps_p, f, "eps_p", dev, numel=pp),
                                           _dev(ws, f, "ws", dev, min_numel=BC_CHECK_WS_DOUBLES), _stream(eps_h)),
               "bc_ccsdt_triples_energy")
    return ws[0]


# ----------------------------------------------------------------------------- checks

def check_sumsq(x: torch.Tensor, ws: Optional[torch.Tensor] = None) -> torch.Tensor:
    """Device scalar sum(x^2) (returned as a 0-d view of the workspace)."""
    if ws is None:
        ws = torch.empty(BC_CHECK_WS_DOUBLES, dtype=torch.float64, device=x.device)
    f, dev = torch.float64, x.device
    with _on(dev):
        _check(lib.bc_check_sumsq(x.numel(), _dev(x, f, "x", dev),
                                  _dev(ws, f, "ws", dev, min_numel=BC_CHECK_WS_DOUBLES), _stream(x)),
               "bc_check_sumsq")
    return ws[0]


def check_energy(ext, t3, eps_h, eps_p, ws=None) -> torch.Tensor:
    if ws is None:
        ws = torch.empty(BC_CHECK_WS_DOUBLES, dtype=torch.float64, device=t3.device)
    f, dev = torch.float64, t3.device
    d = _dims(list(ext[:6]) + [1])
    h = int(ext[0]) + int(ext[1]) + int(ext[2])
    pp = int(ext[3]) + int(ext[4]) + int(ext[5])
    with _on(dev):
        _check(lib.bc_check_energy(ctypes.byref(d), _dev(t3, f, "t3", dev, numel=_n3(ext)),
                                   _dev(eps_h, f, "eps_h", dev, numel=h), _dev(eps_p, f, "eps_p", dev, numel=pp),
                                   _dev(ws, f, "ws", dev, min_numel=BC_CHECK_WS_DOUBLES), _stream(t3)),
               "bc_check_energy")
    return ws[0]


# ----------------------------------------------------------------------------- inputs

KIND_REAL, KIND_INT, KIND_RANGE = 0, 1, 2


def fill(out: torch.Tensor, tensor_id: int, kind: int = KIND_REAL, seed: int = 2015, offset: int = 0,
         lo: float = -1.0, hi: float = 1.0) -> torch.Tensor:
    """Counter-based synthetic values in place (same definition as synthetic/)."""
    if out.dtype == torch.float64:
        fn = lib.bc_fill
    elif out.dtype == torch.float32:
        fn = lib.bc_fill_f32
    else:
        raise TypeError("fill: float64 or float32")
    with _on(out.device):
        _check(fn(int(kind), int(seed), int(tensor_id), int(offset), out.numel(), float(lo), float(hi),
                  _dev(out, out.dtype, "out"), _stream(out)), "bc_fill")
    return out


def probe_fp64_tflops(kind: str, device=None, iters: int = 2000, reps: int = 3) -> float:
    """Measured FP64 throughput (TFLOP/s) of the DFMA ("dfma") or DMMA ("dmma") pipe on
    `device`: best of `reps` timed launches of bc_probe_fp64 (CUDA events)."""
    dev = torch.device("cuda") if device is None else torch.device(device)
    k = {"dfma": 0, "dmma": 1}[kind]
    n = int(lib.bc_probe_scratch_doubles())
    scratch = torch.empty(n, dtype=torch.float64, device=dev)
    flops = ctypes.c_double(0.0)
    st = torch.cuda.current_stream(dev)
    sp = ctypes.c_void_p(st.cuda_stream)
    torch.cuda.set_device(dev)
    _check(lib.bc_probe_fp64(k, 10, _dev(scratch, torch.float64, "scratch"), n, ctypes.byref(flops), sp),
           "bc_probe_fp64")
    best = 0.0
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        _check(lib.bc_probe_fp64(k, iters, scratch.data_ptr(), n, ctypes.byref(flops), sp), "bc_probe_fp64")
        e1.record(st)
        e1.synchronize()
        best = max(best, flops.value / (e0.elapsed_time(e1) * 1e-3) / 1e12)
    return best


def launch_count() -> int:
    return int(lib.bc_launch_count())


def reset_launch_count() -> None:
    lib.bc_reset_launch_count()
