"""Full-size oracle parity for every configuration BASELINE.json names (R21).

The small parity tests run one element group per CTA; these runs are sized so that every
CTA of the persistent grids loops over many groups / units (several waves, a ragged last
group), i.e. the group loop, its prefetch ping-pong and the multi-unit CCSD(T) loops are
compared with the oracle at the sizes the bench's config rows run:

  * cfg 5 spectral sweep: p = 4..12 (and the DMMA sizes p = 7, 14, 15), 3-D sumfact,
    2-D sumfact and local_grad3, N elements with ~64 M points per field (>= 10 waves of
    the grid) + 7, sampled elements (first, last, seeded random) computed one by one by
    the oracle; 1e-12 * S (R14).  fp32 sumfact3d at one p (1e-5 * S).
  * cfg 3/4 tile 24: d1 and d2, all 9 variants fused, random data, 24^3 particle planes
    (13,824 units over the 148-SM grid), every t3 element vs oracle.ccsdt_fused.
  * f4 at full tile 24 (27 variants + energy epilogue) vs the oracle's energy.
"""
import numpy as np
import pytest
import torch

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu

from gpu_util import assert_abs_close, to_dev, to_host  # noqa: E402


@pytest.fixture(scope="module")
def bc():
    import paper_conf_icpp_nelsonrbhhjn15_b200 as m
    return m


def sample(N, n=48, seed=0):
    rng = np.random.default_rng(seed)
    s = set(rng.choice(N, size=n, replace=False).tolist()) | {0, 1, 2, N - 3, N - 2, N - 1}
    return np.array(sorted(s), dtype=np.int64)


def n_for(P1, ndim=3):
    return (1 << 26) // (P1 ** ndim) + 7


@pytest.mark.parametrize("p", [4, 5, 6, 7, 8, 9, 10, 11, 12, 14, 15])
def test_spectral_sweep_3d_sampled(bc, p):
    P1 = p + 1
    N = n_for(P1)
    dev = torch.device("cuda")
    U = bc.fill(torch.empty((N, P1, P1, P1), dtype=torch.float64, device=dev), syn.TID["U"])
    A, B, C = (syn.tensor(syn.TID[n], (P1, P1)) for n in ("A", "B", "C"))
    D = syn.gll_derivative(p)
    V = bc.sumfact3d(to_dev(A), to_dev(B), to_dev(C), U)
    ur, us, ut = bc.local_grad3(to_dev(D), U)
    torch.cuda.synchronize()
    els = sample(N, seed=p)
    idx = torch.from_numpy(els).cuda()
    Uh = syn.elements(syn.TID["U"], P1, els)
    assert np.array_equal(U[idx].cpu().numpy(), Uh)
    assert_abs_close(V[idx].cpu().numpy(), oracle.sumfact3d(A, B, C, Uh),
                     oracle.sumfact3d(abs(A), abs(B), abs(C), abs(Uh)), 1e-12, f"sumfact3d p={p} N={N}")
    for g, r, b, nm in zip((ur, us, ut), oracle.local_grad3(D, Uh), oracle.local_grad3(abs(D), abs(Uh)),
                           ("ur", "us", "ut")):
        assert_abs_close(g[idx].cpu().numpy(), r, b, 1e-12, f"local_grad3 {nm} p={p} N={N}")


@pytest.mark.parametrize("p", [4, 5, 6, 7, 8, 9, 10, 11, 12, 14, 15])
def test_spectral_sweep_2d_sampled(bc, p):
    P1 = p + 1
    N = n_for(P1, 2)
    dev = torch.device("cuda")
    U = bc.fill(torch.empty((N, P1, P1), dtype=torch.float64, device=dev), syn.TID["U"])
    A, B = (syn.tensor(syn.TID[n], (P1, P1)) for n in ("A", "B"))
    V = bc.sumfact2d(to_dev(A), to_dev(B), U)
    torch.cuda.synchronize()
    els = sample(N, n=256, seed=100 + p)
    Uh = syn.elements(syn.TID["U"], P1, els, ndim=2)
    got = V[torch.from_numpy(els).cuda()].cpu().numpy()
    assert_abs_close(got, oracle.sumfact2d(A, B, Uh), oracle.sumfact2d(abs(A), abs(B), abs(Uh)), 1e-12,
                     f"sumfact2d p={p} N={N}")


def test_spectral_f32_full_size_sampled(bc):
    p, P1 = 9, 10
    N = n_for(P1)
    dev = torch.device("cuda")
    U = bc.fill(torch.empty((N, P1, P1, P1), dtype=torch.float32, device=dev), syn.TID["U"])
    A, B, C = (syn.tensor(syn.TID[n], (P1, P1)).astype(np.float32) for n in ("A", "B", "C"))
    V = bc.sumfact3d(*(to_dev(x, torch.float32) for x in (A, B, C)), U)
    torch.cuda.synchronize()
    els = sample(N, seed=7)
    Uh = syn.elements(syn.TID["U"], P1, els).astype(np.float32).astype(np.float64)
    A64, B64, C64 = (x.astype(np.float64) for x in (A, B, C))
    assert_abs_close(V[torch.from_numpy(els).cuda()].cpu().numpy().astype(np.float64),
                     oracle.sumfact3d(A64, B64, C64, Uh), oracle.sumfact3d(abs(A64), abs(B64), abs(C64), abs(Uh)),
                     1e-5, "sumfact3d f32 p=9")


def _ops(family, ext, base):
    h1, h2, h3, p4, p5, p6, k = ext
    na, nb = {"d1": (k * p4 * p5 * h1, h3 * h2 * p6 * k), "d2": (k * p4 * h1 * h2, k * h3 * p6 * p5),
              "s1": (p4 * h1, h3 * h2 * p6 * p5)}[family]
    return ([syn.tensor(base + v, (na,)) for v in range(1, 10)],
            [syn.tensor(base + 20 + v, (nb,)) for v in range(1, 10)])


@pytest.mark.parametrize("family", ["d1", "d2"])
def test_tile24_fused_all9_full(bc, family):
    """24-cube TMA kernel (ccsdt_tma24_kernel): all 9 variants fused, every unit of the
    multi-unit persistent loop compared with the oracle's 9 ascending-v calls."""
    ext = (24,) * 7
    n3 = 24 ** 6
    t3 = syn.tensor(10, (n3,))
    xs, ys = _ops(family, ext, 400 if family == "d1" else 500)
    d3 = to_dev(t3)
    bc.ccsdt_fused(family, ext, d3, [to_dev(x) for x in xs], [to_dev(y) for y in ys])
    ref = oracle.ccsdt_fused(family, ext, t3, xs, ys)
    S = oracle.ccsdt_abs_bound(family, ext, t3, xs, ys)
    assert_abs_close(to_host(d3), ref, S, 1e-12, f"{family} fused tile 24")


def test_f4_tile24_full(bc):
    """f4 (ccsdt_triples24_kernel) at the full tile-24 shape: 27 variants + the energy
    epilogue vs the oracle energy of the t3 built by the 27 oracle calls (bound of
    test_parity_ccsdt.test_triples_energy_f4)."""
    ext = (24,) * 7
    n3 = 24 ** 6
    fams = {f: _ops(f, ext, b) for f, b in (("s1", 600), ("d1", 700), ("d2", 800))}
    eh = syn.tensor(60, (72,), kind=syn.KIND_RANGE, lo=-2.0, hi=-0.5)
    ep = syn.tensor(61, (72,), kind=syn.KIND_RANGE, lo=0.5, hi=2.0)
    t3 = np.zeros(n3)
    S = np.zeros(n3)
    for f in ("s1", "d1", "d2"):
        t3 = oracle.ccsdt_fused(f, ext, t3, *fams[f])
        S += oracle.ccsdt_abs_bound(f, ext, np.zeros(n3), *fams[f])
    E = oracle.energy(ext, t3, eh, ep)
    tol = 2.0 * 1e-12 * abs(oracle.energy(ext, np.sqrt(np.abs(t3) * S), eh, ep)) + 1e-14 * abs(E)
    dv = lambda xs: [to_dev(x) for x in xs]  # noqa: E731
    got = bc.ccsdt_triples_energy(ext, *((dv(fams[f][0]), dv(fams[f][1])) for f in ("s1", "d1", "d2")),
                                  to_dev(eh), to_dev(ep)).item()
    assert abs(got - E) <= tol, (got, E, tol)
