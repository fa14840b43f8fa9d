"""C-ABI boundary checks that need no GPU: the library loads, exports every symbol that
include/barracuda.h declares, and host-side validation rejects bad arguments with the
documented status codes before anything is launched."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "barracuda.h")


@pytest.fixture(scope="module")
def abi():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_icpp_nelsonrbhhjn15_b200 import _abi
    return _abi


def declared_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(bc_[a-z0-9_]+)\s*\(", txt)))


def test_header_declares_entry_points():
    syms = declared_symbols()
    for s in ("bc_sumfact3d", "bc_sumfact2d", "bc_local_grad3", "bc_ccsdt_d1", "bc_ccsdt_d2",
              "bc_ccsdt_d1_fused", "bc_ccsdt_d2_fused", "bc_check_sumsq", "bc_check_energy"):
        assert s in syms


def test_library_exports_every_declared_symbol(abi):
    out = subprocess.run(["nm", "-D", "--defined-only", abi.LIB_PATH], capture_output=True, text=True,
                         check=True).stdout
    exported = set(re.findall(r"\b(bc_[a-z0-9_]+)$", out, flags=re.M))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, f"declared but not exported: {missing}"
    assert set(abi.EXPORTED) == set(declared_symbols())


def test_library_is_sm100a(abi):
    out = subprocess.run(["cuobjdump", "--list-elf", abi.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings(abi):
    for code in (0, -1, -2, -3, -4, -5):
        assert abi.lib.bc_status_string(code)
    assert abi.lib.bc_version() >= 1


# Validation happens before any CUDA call, so these run without a GPU.
FAKE = 1 << 20  # 16-byte aligned fake device addresses: never dereferenced on error paths


def test_spectral_validation(abi):
    L = abi.lib
    a = ctypes.c_void_p
    assert L.bc_sumfact3d(-1, 4, FAKE, FAKE, FAKE, FAKE, FAKE * 4, None) == -1
    assert L.bc_sumfact3d(8, 0, FAKE, FAKE, FAKE, FAKE, FAKE * 4, None) == -1
    assert L.bc_sumfact3d(8, 16, FAKE, FAKE, FAKE, FAKE, FAKE * 4, None) == -4
    assert L.bc_sumfact3d(0, 4, None, None, None, None, None, None) == 0  # N == 0: no-op
    assert L.bc_sumfact3d(8, 4, FAKE, FAKE, FAKE, FAKE + 8, FAKE * 4, None) == -2  # misaligned U
    assert L.bc_sumfact3d(8, 4, FAKE, FAKE, FAKE, FAKE * 4, FAKE * 4, None) == -3  # V aliases U
    assert L.bc_sumfact3d(8, 4, None, FAKE, FAKE, FAKE, FAKE * 4, None) == -1
    assert L.bc_local_grad3(8, 4, FAKE, FAKE * 2, FAKE * 4, FAKE * 4, FAKE * 8, None) == -3  # ur == us
    assert L.bc_sumfact2d(8, 4, FAKE, FAKE, FAKE * 2, FAKE * 2 + 16, None) == -3  # overlap


def test_ccsdt_validation(abi):
    L = abi.lib
    d = abi.TileDims(4, 4, 4, 4, 4, 4, 4)
    assert L.bc_ccsdt_d1(0, ctypes.byref(d), FAKE, FAKE * 2, FAKE * 4, None) == -1
    assert L.bc_ccsdt_d1(10, ctypes.byref(d), FAKE, FAKE * 2, FAKE * 4, None) == -1
    assert L.bc_ccsdt_d2(1, ctypes.byref(d), FAKE, FAKE, FAKE * 4, None) == -3  # t3 aliases t2
    assert L.bc_ccsdt_d2(1, ctypes.byref(d), FAKE + 8, FAKE * 2, FAKE * 4, None) == -2
    bad = abi.TileDims(4, 0, 4, 4, 4, 4, 4)
    assert L.bc_ccsdt_d1(1, ctypes.byref(bad), FAKE, FAKE * 2, FAKE * 4, None) == -1
    big = abi.TileDims(4, 65, 4, 4, 4, 4, 4)
    assert L.bc_ccsdt_d1(1, ctypes.byref(big), FAKE, FAKE * 2, FAKE * 4, None) == -4
    assert L.bc_ccsdt_d1_tile(1, 0, FAKE, FAKE * 2, FAKE * 4, None) == -1
    empty = abi.PtrArray9()
    assert L.bc_ccsdt_d1_fused(ctypes.byref(d), FAKE, empty, empty, None) == 0  # nothing to do
    # fused family + energy check: family range, ws required, eps required, ws must not alias t3
    assert L.bc_ccsdt_fused_energy(0, ctypes.byref(d), FAKE, empty, empty, FAKE * 8, FAKE * 9, FAKE * 10, None) == -1
    assert L.bc_ccsdt_fused_energy(4, ctypes.byref(d), FAKE, empty, empty, FAKE * 8, FAKE * 9, FAKE * 10, None) == -1
    assert L.bc_ccsdt_fused_energy(2, ctypes.byref(d), FAKE, empty, empty, FAKE * 8, FAKE * 9, None, None) == -1
    assert L.bc_ccsdt_fused_energy(2, ctypes.byref(d), FAKE, empty, empty, None, FAKE * 9, FAKE * 10, None) == -1
    assert L.bc_ccsdt_fused_energy(2, ctypes.byref(d), FAKE, empty, empty, FAKE * 8, FAKE * 9, FAKE, None) == -3


def test_python_binding_refuses_cpu_tensors(abi):
    import torch
    import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
    A = torch.eye(3, dtype=torch.float64)
    U = torch.zeros(2, 3, 3, 3, dtype=torch.float64)
    with pytest.raises(ValueError, match="CUDA"):
        bc.sumfact3d(A, A, A, U, out=U.clone())
