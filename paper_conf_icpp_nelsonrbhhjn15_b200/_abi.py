"""ctypes declarations of include/barracuda.h (libbarracuda.so, built in-tree).

There is no fallback: if the shared library is missing or fails to load, importing this
module raises.  Build it with `python -c "import __graft_entry__ as g; g.build()"`.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BARRACUDA_LIB") or os.path.join(_HERE, "libbarracuda.so")  # override: variant sweeps

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"libbarracuda.so not found at {LIB_PATH}: build it first (__graft_entry__.build()); "
        "there is no CPU fallback")

lib = ctypes.CDLL(LIB_PATH)

_vp, _i64, _i32, _u64, _d = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double


class TileDims(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in ("h1", "h2", "h3", "p4", "p5", "p6", "k")]


PtrArray9 = _vp * 9

_SIGS = {
    "bc_sumfact3d": [_i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp],
    "bc_sumfact3d_check": [_i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp, _vp],
    "bc_sumfact3d_f32": [_i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp],
    "bc_sumfact2d": [_i64, _i32, _vp, _vp, _vp, _vp, _vp],
    "bc_local_grad3": [_i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp],
    "bc_local_grad3_t": [_i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp],
    "bc_ax_e": [_i64, _i32, _vp, _vp, _vp, _vp, _vp],
    "bc_ccsdt_d1": [_i32, ctypes.POINTER(TileDims), _vp, _vp, _vp, _vp],
    "bc_ccsdt_d2": [_i32, ctypes.POINTER(TileDims), _vp, _vp, _vp, _vp],
    "bc_ccsdt_s1": [_i32, ctypes.POINTER(TileDims), _vp, _vp, _vp, _vp],
    "bc_ccsdt_d1_fused": [ctypes.POINTER(TileDims), _vp, PtrArray9, PtrArray9, _vp],
    "bc_ccsdt_d2_fused": [ctypes.POINTER(TileDims), _vp, PtrArray9, PtrArray9, _vp],
    "bc_ccsdt_s1_fused": [ctypes.POINTER(TileDims), _vp, PtrArray9, PtrArray9, _vp],
    "bc_ccsdt_fused_energy": [_i32, ctypes.POINTER(TileDims), _vp, PtrArray9, PtrArray9, _vp, _vp, _vp, _vp],
    "bc_ccsdt_triples_energy": [ctypes.POINTER(TileDims), PtrArray9, PtrArray9, PtrArray9, PtrArray9, PtrArray9,
                                PtrArray9, _vp, _vp, _vp, _vp],
    "bc_ccsdt_d1_tile": [_i32, _i32, _vp, _vp, _vp, _vp],
    "bc_ccsdt_d2_tile": [_i32, _i32, _vp, _vp, _vp, _vp],
    "bc_check_sumsq": [_i64, _vp, _vp, _vp],
    "bc_check_energy": [ctypes.POINTER(TileDims), _vp, _vp, _vp, _vp, _vp],
    "bc_fill": [_i32, _u64, _u64, _u64, _i64, _d, _d, _vp, _vp],
    "bc_fill_f32": [_i32, _u64, _u64, _u64, _i64, _d, _d, _vp, _vp],
    "bc_probe_fp64": [_i32, _i32, _vp, _i64, ctypes.POINTER(_d), _vp],
    "bc_probe_scratch_doubles": [],
    "bc_status_string": [_i32],
    "bc_last_cuda_error": [],
    "bc_version": [],
    "bc_launch_count": [],
    "bc_reset_launch_count": [],
}

EXPORTED = tuple(_SIGS)

for _name, _args in _SIGS.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = _i32
lib.bc_status_string.restype = ctypes.c_char_p
lib.bc_launch_count.restype = _i64
lib.bc_probe_scratch_doubles.restype = _i64
lib.bc_reset_launch_count.restype = None

BC_CHECK_WS_DOUBLES = 1024
BC_MAX_P = 15
BC_MAX_TILE_EXTENT = 64
