"""Stress gate for the warp-specialised TMA element-ring kernels (csrc/spectral.cu:
sumfact_tma_kernel 3-D/2-D, local_grad3_tma_kernel).

The rings' synchronisation (full/empty/done mbarriers, NG consumer groups sharing NB slots,
bulk copies completing out of order) is exercised at sizes where every CTA cycles its ring
hundreds of times: each kernel runs REPEATS times on the same integer-valued inputs and
every run must be bitwise identical to the first (device-side comparison of whole
outputs), and sampled elements bitwise equal to the oracle (integer data: exact sums).
A parity wait that aliased a ring phase showed up here as wrong bytes or as an
'unspecified launch failure' at large N."""
import numpy as np
import pytest
import torch

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu

REPEATS = 12


@pytest.fixture(scope="module")
def bc():
    import paper_conf_icpp_nelsonrbhhjn15_b200 as m
    return m


def int_field(bc, shape, tid):
    return bc.fill(torch.empty(shape, dtype=torch.float64, device="cuda"), tid, kind=bc.KIND_INT)


def sample(N, seed):
    rng = np.random.default_rng(seed)
    return np.array(sorted(set(rng.choice(N, size=24, replace=False).tolist()) | {0, N - 1}), dtype=np.int64)


def int_elements(tid, P1, els, ndim=3):
    return syn.elements(tid, P1, els, ndim=ndim, kind=syn.KIND_INT)


def repeat_equal(fn, outs):
    ref = [o.clone() for o in outs]
    for r in range(REPEATS):
        for o in outs:
            o.fill_(float("nan"))
        fn()
        torch.cuda.synchronize()
        for o, x in zip(outs, ref):
            assert torch.equal(o, x), f"repeat {r} differs"
    return ref


@pytest.mark.parametrize("P1", [5, 9, 13])
def test_ring_sumfact3d_repeat_bitwise(bc, P1):
    N = (1 << 28) // (P1 ** 3 * 8) + 1
    A, B, C = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3, 4))
    dA, dB, dC = (torch.from_numpy(x).cuda() for x in (A, B, C))
    U = int_field(bc, (N, P1, P1, P1), syn.TID["U"])
    V = torch.empty_like(U)
    bc.sumfact3d(dA, dB, dC, U, out=V)
    torch.cuda.synchronize()
    (Vr,) = repeat_equal(lambda: bc.sumfact3d(dA, dB, dC, U, out=V), [V])
    els = sample(N, P1)
    got = Vr[torch.from_numpy(els).cuda()].cpu().numpy()
    assert np.array_equal(got, oracle.sumfact3d(A, B, C, int_elements(syn.TID["U"], P1, els)))


@pytest.mark.parametrize("P1", [5, 9, 13])
def test_ring_sumfact2d_repeat_bitwise(bc, P1):
    N = (1 << 28) // (P1 ** 2 * 8) + 3
    A, B = (syn.tensor(t, (P1, P1), kind=syn.KIND_INT) for t in (2, 3))
    dA, dB = (torch.from_numpy(x).cuda() for x in (A, B))
    U = int_field(bc, (N, P1, P1), syn.TID["U"])
    V = torch.empty_like(U)
    bc.sumfact2d(dA, dB, U, out=V)
    torch.cuda.synchronize()
    (Vr,) = repeat_equal(lambda: bc.sumfact2d(dA, dB, U, out=V), [V])
    els = sample(N, 10 + P1)
    got = Vr[torch.from_numpy(els).cuda()].cpu().numpy()
    assert np.array_equal(got, oracle.sumfact2d(A, B, int_elements(syn.TID["U"], P1, els, ndim=2)))


@pytest.mark.parametrize("P1", [5, 9, 13])
def test_ring_local_grad3_repeat_bitwise(bc, P1):
    N = (1 << 28) // (P1 ** 3 * 8) + 1
    D = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    dD = torch.from_numpy(D).cuda()
    U = int_field(bc, (N, P1, P1, P1), syn.TID["U"])
    outs = tuple(torch.empty_like(U) for _ in range(3))
    bc.local_grad3(dD, U, out=outs)
    torch.cuda.synchronize()
    refs = repeat_equal(lambda: bc.local_grad3(dD, U, out=outs), list(outs))
    els = sample(N, 20 + P1)
    idx = torch.from_numpy(els).cuda()
    for g, r in zip(refs, oracle.local_grad3(D, int_elements(syn.TID["U"], P1, els))):
        assert np.array_equal(g[idx].cpu().numpy(), r)


@pytest.mark.parametrize("P1", [5, 9, 13])
def test_ring_local_grad3_t_repeat_bitwise(bc, P1):
    N = (1 << 27) // (P1 ** 3 * 8) + 1
    D = syn.tensor(6, (P1, P1), kind=syn.KIND_INT)
    dD = torch.from_numpy(D).cuda()
    ins = [int_field(bc, (N, P1, P1, P1), t) for t in (7, 8, 9)]
    U = torch.empty_like(ins[0])
    bc.local_grad3_t(dD, *ins, out=U)
    torch.cuda.synchronize()
    (Ur,) = repeat_equal(lambda: bc.local_grad3_t(dD, *ins, out=U), [U])
    els = sample(N, 30 + P1)
    got = Ur[torch.from_numpy(els).cuda()].cpu().numpy()
    ref = oracle.local_grad3_t(D, *(int_elements(t, P1, els) for t in (7, 8, 9)))
    assert np.array_equal(got, ref)
