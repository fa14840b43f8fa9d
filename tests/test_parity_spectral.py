"""GPU parity of the spectral family (through the C ABI) against the CPU oracle.

Integer data in [-4,3]: every partial sum is exact, so results must be BITWISE equal.
Uniform [-1,1) data: componentwise |gpu - oracle| <= 1e-12 * S (fp64), 1e-5 * S (fp32),
S = abs-value evaluation (R14).  Outputs are pre-poisoned with NaN so an
unwritten point fails.  N covers 1, odd, the per-CTA group size +/- 1 and several groups.
"""
import numpy as np
import pytest
import torch

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu

from gpu_util import assert_abs_close, poisoned_like, to_dev, to_host  # noqa: E402


@pytest.fixture(scope="module")
def bc():
    import paper_conf_icpp_nelsonrbhhjn15_b200 as m
    assert torch.cuda.is_available()
    return m


def Ns_for(P1):
    # elements per CTA group E (Cfg in csrc/spectral.cu): 36 KiB / padded element size, made even.
    # N < 128 runs the shared-memory-operator kernels, N >= 128 the constant-bank ones
    # (OPS_CONST_MIN_N in csrc/spectral.cu): both paths at every P1
    return [1, 2, 3, 37, 130]


ALL_P1 = list(range(2, 17))


@pytest.mark.parametrize("P1", ALL_P1)
def test_sumfact3d_integer_bitwise(bc, P1):
    A, B, C = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3, 4))
    for N in Ns_for(P1):
        U = syn.tensor(1, (N, P1, P1, P1), kind=syn.KIND_INT)
        Ud = to_dev(U)
        V = bc.sumfact3d(to_dev(A), to_dev(B), to_dev(C), Ud, out=poisoned_like(Ud))
        assert np.array_equal(to_host(V), oracle.sumfact3d(A, B, C, U)), f"P1={P1} N={N}"


@pytest.mark.parametrize("N", [67, 257])
@pytest.mark.parametrize("P1", ALL_P1)
def test_sumfact3d_random_tolerance(bc, P1, N):
    A, B, C = (syn.tensor(t, (P1, P1)) for t in (2, 3, 4))
    U = syn.tensor(1, (N, P1, P1, P1))
    Ud = to_dev(U)
    V = bc.sumfact3d(to_dev(A), to_dev(B), to_dev(C), Ud, out=poisoned_like(Ud))
    S = oracle.sumfact3d(abs(A), abs(B), abs(C), abs(U))
    assert_abs_close(to_host(V), oracle.sumfact3d(A, B, C, U), S, 1e-12, f"sumfact3d P1={P1}")


@pytest.mark.parametrize("P1", [2, 5, 8, 13, 16])
def test_sumfact3d_f32(bc, P1):
    N = 45
    A, B, C = (syn.tensor(t, (P1, P1)).astype(np.float32) for t in (2, 3, 4))
    U = syn.tensor(1, (N, P1, P1, P1)).astype(np.float32)
    Ud = to_dev(U, torch.float32)
    V = bc.sumfact3d(*(to_dev(x, torch.float32) for x in (A, B, C)), Ud, out=poisoned_like(Ud))
    A64, B64, C64, U64 = (x.astype(np.float64) for x in (A, B, C, U))
    S = oracle.sumfact3d(abs(A64), abs(B64), abs(C64), abs(U64))
    assert_abs_close(to_host(V), oracle.sumfact3d(A64, B64, C64, U64), S, 1e-5, f"sumfact3d_f32 P1={P1}")


@pytest.mark.parametrize("P1", ALL_P1)
def test_sumfact2d(bc, P1):
    A, B = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3))
    for N in (1, 3, 255, 1001):
        U = syn.tensor(1, (N, P1, P1), kind=syn.KIND_INT)
        Ud = to_dev(U)
        V = bc.sumfact2d(to_dev(A), to_dev(B), Ud, out=poisoned_like(Ud))
        assert np.array_equal(to_host(V), oracle.sumfact2d(A, B, U)), f"P1={P1} N={N}"
    A, B = (syn.tensor(t, (P1, P1)) for t in (2, 3))
    U = syn.tensor(1, (333, P1, P1))
    V = bc.sumfact2d(to_dev(A), to_dev(B), to_dev(U))
    assert_abs_close(to_host(V), oracle.sumfact2d(A, B, U), oracle.sumfact2d(abs(A), abs(B), abs(U)), 1e-12)


@pytest.mark.parametrize("P1", ALL_P1)
def test_local_grad3(bc, P1):
    D = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    for N in (1, 3, 37, 130):
        U = syn.tensor(1, (N, P1, P1, P1), kind=syn.KIND_INT)
        Ud = to_dev(U)
        outs = tuple(poisoned_like(Ud) for _ in range(3))
        got = bc.local_grad3(to_dev(D), Ud, out=outs)
        for g, r, name in zip(got, oracle.local_grad3(D, U), ("ur", "us", "ut")):
            assert np.array_equal(to_host(g), r), f"{name} P1={P1} N={N}"
    Dg = syn.gll_derivative(P1 - 1)
    for N in (29, 131):
        U = syn.tensor(1, (N, P1, P1, P1))
        got = bc.local_grad3(to_dev(Dg), to_dev(U))
        for g, r, b in zip(got, oracle.local_grad3(Dg, U), oracle.local_grad3(abs(Dg), abs(U))):
            assert_abs_close(to_host(g), r, b, 1e-12, f"local_grad3 P1={P1} N={N}")


@pytest.mark.parametrize("P1", ALL_P1)
def test_local_grad3_t(bc, P1):
    D = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    for N in (11, 150):  # shared-memory and constant-bank operator kernels
        ur, us, ut = (syn.tensor(t, (N, P1, P1, P1), kind=syn.KIND_INT) for t in (7, 8, 9))
        got = bc.local_grad3_t(to_dev(D), to_dev(ur), to_dev(us), to_dev(ut), out=poisoned_like(to_dev(ur)))
        assert np.array_equal(to_host(got), oracle.local_grad3_t(D, ur, us, ut)), f"P1={P1} N={N}"


@pytest.mark.parametrize("N", [7, 140])
@pytest.mark.parametrize("P1", [2, 5, 8, 9, 12, 13, 16])
def test_ax_e(bc, P1, N):
    D = syn.gll_derivative(P1 - 1)
    U = syn.tensor(1, (N, P1, P1, P1))
    G = syn.tensor(11, (N, 6, P1, P1, P1))
    got = bc.ax_e(to_dev(D), to_dev(U), to_dev(G), out=poisoned_like(to_dev(U)))
    ref = oracle.ax_e(D, U, G)
    S = oracle.ax_e(abs(D), abs(U), abs(G))
    assert_abs_close(to_host(got), ref, S, 1e-12, f"ax_e P1={P1}")
    Di = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    Ui = syn.tensor(1, (N, P1, P1, P1), kind=syn.KIND_INT)
    Gi = syn.tensor(11, (N, 6, P1, P1, P1), kind=syn.KIND_INT)
    assert np.array_equal(to_host(bc.ax_e(to_dev(Di), to_dev(Ui), to_dev(Gi))), oracle.ax_e(Di, Ui, Gi))


def test_paper_form_through_gpu(bc):
    """Eq. (1) exactly as printed (V[i j k] += A[l k] B[m j] C[n i] U[l m n]) at the paper's
    size 10 via reading R1, bitwise on integers."""
    P1 = 10
    A, B, C = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3, 4))
    U = syn.tensor(1, (P1, P1, P1), kind=syn.KIND_INT)
    ref = np.einsum("lk,mj,ni,lmn->ijk", A, B, C, U)
    got = bc.sumfact3d(to_dev(A.T.copy()), to_dev(B.T.copy()), to_dev(C.T.copy()), to_dev(U.transpose(2, 1, 0)[None]))
    assert np.array_equal(to_host(got)[0], ref)


def test_device_fill_matches_synthetic_bitwise(bc):
    for kind, lo, hi in ((syn.KIND_REAL, -1, 1), (syn.KIND_INT, -1, 1), (syn.KIND_RANGE, -2.0, -0.5)):
        for off in (0, 12345):
            t = torch.empty(100003, dtype=torch.float64, device="cuda")
            bc.fill(t, 7, kind=kind, offset=off, lo=lo, hi=hi)
            ref = syn.values(7, np.arange(off, off + 100003, dtype=np.uint64), kind=kind, lo=lo, hi=hi)
            assert np.array_equal(to_host(t), ref)
    t = torch.empty(1000, dtype=torch.float32, device="cuda")
    bc.fill(t, 3)
    assert np.array_equal(t.cpu().numpy(), syn.tensor(3, (1000,)).astype(np.float32))


def test_check_sumsq(bc):
    x = syn.tensor(1, (1234567,))
    got = float(bc.check_sumsq(to_dev(x)).item())
    ref = oracle.sumsq(x)
    assert abs(got - ref) <= 1e-12 * ref


def test_errors_raise(bc):
    A = torch.eye(5, dtype=torch.float64, device="cuda")
    U = torch.zeros(3, 5, 5, 5, dtype=torch.float64, device="cuda")
    with pytest.raises(bc.BarracudaError, match="ALIAS"):
        bc.sumfact3d(A, A, A, U, out=U)


@pytest.mark.parametrize("P1", [2, 5, 13, 16])
def test_sumfact3d_fused_check_scalar(bc, P1):
    """bc_sumfact3d_check: V as bc_sumfact3d, plus ws[0] = sum V^2 from the store epilogue."""
    A, B, C = (syn.tensor(t, (P1, P1)) for t in (2, 3, 4))
    U = syn.tensor(1, (301, P1, P1, P1))
    ws = torch.full((1024,), float("nan"), dtype=torch.float64, device="cuda")
    V = bc.sumfact3d(to_dev(A), to_dev(B), to_dev(C), to_dev(U), check_ws=ws)
    Vr = oracle.sumfact3d(A, B, C, U)
    assert_abs_close(to_host(V), Vr, oracle.sumfact3d(abs(A), abs(B), abs(C), abs(U)), 1e-12, "V")
    ref = oracle.sumsq(Vr)
    assert abs(ws[0].item() - ref) <= 1e-12 * ref


def test_constant_bank_operators_two_streams_and_graph(bc):
    """The constant-bank operator slots (csrc/spectral.cu, N >= 128) under concurrency:
    calls with DIFFERENT operators queued alternately on two streams, more calls than
    slots, each result equal (bitwise, integer data) to the oracle with its own operators;
    then the same calls captured into a CUDA graph and replayed."""
    P1, N = 13, 160
    U = syn.tensor(1, (N, P1, P1, P1), kind=syn.KIND_INT)
    Ud = to_dev(U)
    ops = [[syn.tensor(200 + 3 * i + j, (P1, P1), kind=syn.KIND_INT) for j in range(3)] for i in range(6)]
    refs = [oracle.sumfact3d(*o, U) for o in ops]
    dops = [[to_dev(x) for x in o] for o in ops]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    outs = [poisoned_like(Ud) for _ in ops]
    torch.cuda.synchronize()
    for i, (o, out) in enumerate(zip(dops, outs)):
        with torch.cuda.stream(streams[i % 2]):
            bc.sumfact3d(*o, Ud, out=out)
    torch.cuda.synchronize()
    for i, (out, ref) in enumerate(zip(outs, refs)):
        assert np.array_equal(to_host(out), ref), f"call {i} (stream {i % 2})"
    g = torch.cuda.CUDAGraph()
    gouts = [poisoned_like(Ud) for _ in ops]
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            for o, out in zip(dops, gouts):
                bc.sumfact3d(*o, Ud, out=out)
    g.replay()
    torch.cuda.synchronize()
    for i, (out, ref) in enumerate(zip(gouts, refs)):
        assert np.array_equal(to_host(out), ref), f"graph call {i}"


@pytest.mark.parametrize("P1", [13])
def test_sumfact3d_tma_ring_integer_bitwise(bc, P1):
    """The warp-specialised TMA element-ring kernel (csrc/spectral.cu sumfact3d_tma_kernel,
    odd P1 >= 9, N >= 128, 16-byte aligned U): N = 148 CTAs x 2 elements x 6 slots x 2 + 1,
    so every CTA's ring wraps at least twice and the last item is ragged (one element, an
    odd number of values: bulk copy + the plain-copied last value); every element bitwise
    vs the oracle (items alternately start on and 8 bytes off a 16-byte boundary); then
    N + 1 elements (even: no plain-copied value) with the fused check scalar."""
    A, B, C = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3, 4))
    N = 148 * 2 * 6 * 2 + 1
    U = syn.tensor(1, (N + 1, P1, P1, P1), kind=syn.KIND_INT)
    Ud = to_dev(U)
    Ad, Bd, Cd = to_dev(A), to_dev(B), to_dev(C)
    ref = oracle.sumfact3d(A, B, C, U)
    V = bc.sumfact3d(Ad, Bd, Cd, Ud[:N], out=poisoned_like(Ud[:N]))
    assert np.array_equal(to_host(V), ref[:N]), f"P1={P1} N={N}"
    ws = torch.full((1024,), float("nan"), dtype=torch.float64, device="cuda")
    V2 = bc.sumfact3d(Ad, Bd, Cd, Ud, out=poisoned_like(Ud), check_ws=ws)
    assert np.array_equal(to_host(V2), ref)
    s = oracle.sumsq(ref)
    assert abs(ws[0].item() - s) <= 1e-12 * s


@pytest.mark.parametrize("N", [128, 129, 148 * 2 * 5 * 2 + 1, 148 * 2 * 5 * 3 + 2])
def test_local_grad3_tma_ring_integer_bitwise(bc, N):
    """The warp-specialised TMA element-ring local_grad3 (csrc/spectral.cu
    local_grad3_tma_kernel, P1 = 13, N >= 128, 16-byte aligned U and ur): rings that do not
    wrap, wrap twice and three times; items alternately on and 8 bytes off a 16-byte
    boundary, so ur's bulk store writes its first/last value by plain stores; an odd N
    (the last item's final value plain-copied in); ur/us/ut every element bitwise."""
    P1 = 13
    D = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    U = syn.tensor(1, (N, P1, P1, P1), kind=syn.KIND_INT)
    Ud = to_dev(U)
    outs = tuple(poisoned_like(Ud) for _ in range(3))
    got = bc.local_grad3(to_dev(D), Ud, out=outs)
    for g, r, name in zip(got, oracle.local_grad3(D, U), ("ur", "us", "ut")):
        assert np.array_equal(to_host(g), r), f"{name} N={N}"


@pytest.mark.parametrize("P1", [5, 9, 13])
@pytest.mark.parametrize("N", [128, 148 * 40 * 12 * 2 + 1])
def test_sumfact2d_tma_ring_integer_bitwise(bc, P1, N):
    """The TMA element-ring sumfact2d (csrc/spectral.cu sumfact_tma_kernel<P1, 1>, items of
    32 NWG R / P1 2-D elements, where enabled; the other P1 run the unbuffered kernel): a
    ring that does not wrap and one that wraps at least twice with a ragged last item; every
    element bitwise vs the oracle."""
    A, B = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3))
    U = syn.tensor(1, (N, P1, P1), kind=syn.KIND_INT)
    Ud = to_dev(U)
    V = bc.sumfact2d(to_dev(A), to_dev(B), Ud, out=poisoned_like(Ud))
    assert np.array_equal(to_host(V), oracle.sumfact2d(A, B, U)), f"P1={P1} N={N}"


@pytest.mark.parametrize("P1", [5, 9, 11, 13])
def test_local_grad3_t_tma_ring_integer_bitwise(bc, P1):
    """The TMA ring local_grad3_t (csrc/spectral.cu local_grad3_t_tma_kernel: three input
    fields per slot): N large enough for every CTA's 4-slot ring to wrap several times, odd
    (ragged last item with plain-copied final values); every element bitwise."""
    N = 148 * 4 * 3 * max(1, 192 // (P1 * P1)) + 1
    D = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    ur, us, ut = (syn.tensor(t, (N, P1, P1, P1), kind=syn.KIND_INT) for t in (7, 8, 9))
    got = bc.local_grad3_t(to_dev(D), to_dev(ur), to_dev(us), to_dev(ut), out=poisoned_like(to_dev(ur)))
    assert np.array_equal(to_host(got), oracle.local_grad3_t(D, ur, us, ut)), f"P1={P1} N={N}"
