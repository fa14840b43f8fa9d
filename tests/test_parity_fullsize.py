"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(workload.Step: local_grad3 / sumfact3d p=12 on N=262,144 elements, sumfact2d on the same
batch, CCSD(T) d1+d2 fused tile 16 x 8 blocks, check scalars), checked on sampled outputs
the oracle computes one by one (first, last and seeded random elements; first and last
CCSD(T) blocks in full) and on the full check scalars (R21)."""
import numpy as np
import pytest
import torch

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu

from gpu_util import assert_abs_close  # noqa: E402


@pytest.fixture(scope="module")
def step():
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import Step, StepConfig
    st = Step(StepConfig(), rank=0, world=1, device=torch.device("cuda"))
    st.t3_init = [t.detach().cpu().numpy().copy() for t in st.t3]
    st.run()
    torch.cuda.synchronize()
    return st


def test_spectral_sampled(step):
    c = step.cfg
    P1 = c.P1
    els = step.sample_elements(64)
    U = syn.elements(syn.TID["U"], P1, els)
    A, B, C = (syn.tensor(syn.TID[n], (P1, P1)) for n in ("A", "B", "C"))
    D = syn.gll_derivative(c.p)
    idx = torch.from_numpy(els).cuda()
    assert np.array_equal(step.U[idx].cpu().numpy(), U)  # device generator == host generator
    ref = oracle.local_grad3(D, U)
    bnd = oracle.local_grad3(abs(D), abs(U))
    for got, r, b, name in zip((step.ur, step.us, step.ut), ref, bnd, ("ur", "us", "ut")):
        assert_abs_close(got[idx].cpu().numpy(), r, b, 1e-12, name)
    assert_abs_close(step.V[idx].cpu().numpy(), oracle.sumfact3d(A, B, C, U),
                     oracle.sumfact3d(abs(A), abs(B), abs(C), abs(U)), 1e-12, "sumfact3d")
    U2 = U.reshape(-1, P1, P1)
    got2 = step.V2.view(c.n_elem, P1, P1, P1)[idx].cpu().numpy().reshape(-1, P1, P1)
    assert_abs_close(got2, oracle.sumfact2d(A, B, U2), oracle.sumfact2d(abs(A), abs(B), abs(U2)), 1e-12,
                     "sumfact2d")


def test_ccsdt_blocks_and_checks(step):
    c = step.cfg
    ext = step.ext
    V = step.V.cpu().numpy()
    ref_sumsq = oracle.sumsq(V)
    assert abs(step.checks[0].item() - ref_sumsq) <= 1e-12 * ref_sumsq
    eh, ep = step.eps_h.cpu().numpy(), step.eps_p.cpu().numpy()
    E = 0.0
    for b in range(c.blocks):
        t3 = step.t3[b].cpu().numpy()
        E += oracle.energy(ext, t3, eh, ep)
        if b in (0, c.blocks - 1):
            ref = step.t3_init[b]
            bound = np.abs(ref)
            for fam in c.families:
                t2s = [x.cpu().numpy() for x in step.t2[(fam, b)]]
                v2s = [x.cpu().numpy() for x in step.v2[(fam, b)]]
                bound = bound + oracle.ccsdt_abs_bound(fam, ext, np.zeros_like(ref), t2s, v2s)
                ref = oracle.ccsdt_fused(fam, ext, ref, t2s, v2s)
            assert_abs_close(t3, ref, bound, 1e-12, f"t3 block {b}")
    assert abs(step.checks[1].item() - E) <= 1e-12 * abs(E)
