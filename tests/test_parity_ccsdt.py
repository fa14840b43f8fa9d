"""GPU parity of the CCSD(T) family (through the C ABI) against the oracle's literal
7-deep loops.  Integer data with unequal extents (all 7 distinct) must be bitwise equal —
a swapped extent or index cannot hide.  t3 starts non-zero (accumulate semantics)."""
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


def sizes(family, ext):
    h1, h2, h3, p4, p5, p6, k = ext
    if family == "d1":
        return k * p4 * p5 * h1, h3 * h2 * p6 * k
    if family == "d2":
        return k * p4 * h1 * h2, k * h3 * p6 * p5
    return p4 * h1, h3 * h2 * p6 * p5


def n3(ext):
    return int(np.prod(ext[:6]))


# includes shapes that take the 16-cube tensor-core (DMMA) path: hole extents 16/32/30 with
# even k (ragged k chunk: 6, 10) and a ragged cube edge (30), and odd k (falls back to DFMA);
# 16^3 / 24^3 holes with k <= 32 take the single-variant streaming kernel (ccsdt_svs_kernel):
# unequal particle extents (A-name-major unit order), k = 1, 2, 7, 10, 16, 24, 32, one plane
EXTS = [(3, 4, 5, 6, 2, 7, 3), (9, 17, 13, 5, 3, 4, 19), (8, 8, 8, 8, 8, 8, 8), (1, 1, 1, 1, 1, 1, 1),
        (16, 32, 16, 3, 4, 2, 6), (30, 16, 16, 2, 3, 2, 10), (16, 16, 30, 2, 2, 3, 10), (16, 16, 16, 2, 3, 2, 7),
        (16, 16, 16, 3, 2, 4, 16), (16, 16, 16, 2, 4, 3, 32), (24, 24, 24, 2, 3, 2, 10), (24, 24, 24, 3, 1, 2, 24),
        (16, 16, 16, 1, 1, 1, 1), (16, 16, 16, 1, 2, 1, 2)]


@pytest.mark.parametrize("family", ["d1", "d2", "s1"])
@pytest.mark.parametrize("ext", EXTS)
def test_single_variant_integer_bitwise(bc, family, ext):
    na, nb = sizes(family, ext)
    for v in range(1, 10):
        t3 = syn.tensor(10, (n3(ext),), kind=syn.KIND_INT)
        t2 = syn.tensor(20 + v, (na,), kind=syn.KIND_INT)
        v2 = syn.tensor(40 + v, (nb,), kind=syn.KIND_INT)
        d3 = to_dev(t3)
        bc.ccsdt(family, v, ext, d3, to_dev(t2), to_dev(v2))
        assert np.array_equal(to_host(d3), oracle.ccsdt(family, v, ext, t3, t2, v2)), f"{family}_{v} ext={ext}"


@pytest.mark.parametrize("family", ["d1", "d2", "s1"])
@pytest.mark.parametrize("ext", [(3, 4, 5, 6, 2, 7, 3), (12, 12, 12, 7, 7, 7, 21), (5, 5, 5, 3, 3, 3, 40),
                                 (16, 16, 16, 3, 3, 3, 4), (24, 24, 24, 2, 2, 2, 4)])
def test_fused_integer_bitwise(bc, family, ext):
    na, nb = sizes(family, ext)
    t3 = syn.tensor(10, (n3(ext),), kind=syn.KIND_INT)
    t2s = [syn.tensor(20 + v, (na,), kind=syn.KIND_INT) for v in range(1, 10)]
    v2s = [syn.tensor(40 + v, (nb,), kind=syn.KIND_INT) for v in range(1, 10)]
    for mask in (range(1, 10), (2, 5, 9), (7,)):
        a = [t2s[v - 1] if v in mask else None for v in range(1, 10)]
        d3 = to_dev(t3)
        bc.ccsdt_fused(family, ext, d3, [None if x is None else to_dev(x) for x in a], [to_dev(x) for x in v2s])
        assert np.array_equal(to_host(d3), oracle.ccsdt_fused(family, ext, t3, a, v2s)), f"{family} mask={list(mask)}"


# hole extents in (16, 24] take the 24-cube TMA path (ccsdt_tma24_kernel): unequal holes, a
# ragged k chunk (10 = 4 + 4 + 2), a second ragged cube (40 = 24 + 16), exact 24-cubes
# (24, 24, 24, ...) is a dense block (contiguous t3 runs per unit, division-free seed/store)
EXTS24 = [(18, 22, 24, 3, 2, 4, 10), (24, 24, 40, 2, 2, 3, 8), (24, 20, 22, 2, 3, 2, 6), (24, 24, 24, 2, 3, 2, 10)]


@pytest.mark.parametrize("family", ["d1", "d2"])
@pytest.mark.parametrize("ext", EXTS24)
def test_tile24_path_integer_bitwise(bc, family, ext):
    na, nb = sizes(family, ext)
    t3 = syn.tensor(10, (n3(ext),), kind=syn.KIND_INT)
    t2s = [syn.tensor(20 + v, (na,), kind=syn.KIND_INT) for v in range(1, 10)]
    v2s = [syn.tensor(40 + v, (nb,), kind=syn.KIND_INT) for v in range(1, 10)]
    for v in (1, 2, 3, 5, 9):
        d3 = to_dev(t3)
        bc.ccsdt(family, v, ext, d3, to_dev(t2s[v - 1]), to_dev(v2s[v - 1]))
        assert np.array_equal(to_host(d3), oracle.ccsdt(family, v, ext, t3, t2s[v - 1], v2s[v - 1])), f"{family}_{v}"
    for mask in (range(1, 10), (2, 4, 9)):
        a = [t2s[v - 1] if v in mask else None for v in range(1, 10)]
        d3 = to_dev(t3)
        bc.ccsdt_fused(family, ext, d3, [None if x is None else to_dev(x) for x in a], [to_dev(x) for x in v2s])
        assert np.array_equal(to_host(d3), oracle.ccsdt_fused(family, ext, t3, a, v2s)), f"{family} mask={list(mask)}"


@pytest.mark.parametrize("family", ["d1", "d2"])
@pytest.mark.parametrize("tile", [16, 24])
def test_tile_random_tolerance(bc, family, tile):
    """North-star tile sizes (16; BASELINE: 24), uniform data, rtol 1e-12 of S."""
    ext = (tile,) * 7
    na, nb = sizes(family, ext)
    t3 = syn.tensor(10, (n3(ext),))
    t2s = [syn.tensor(20 + v, (na,)) for v in range(1, 10)]
    v2s = [syn.tensor(40 + v, (nb,)) for v in range(1, 10)]
    if tile == 16:  # fused over all 9 (the oracle's 9 literal passes take too long at 24)
        d3 = to_dev(t3)
        bc.ccsdt_fused(family, ext, d3, [to_dev(x) for x in t2s], [to_dev(x) for x in v2s])
        ref = oracle.ccsdt_fused(family, ext, t3, t2s, v2s)
        S = oracle.ccsdt_abs_bound(family, ext, t3, t2s, v2s)
        assert_abs_close(to_host(d3), ref, S, 1e-12, f"{family} fused tile {tile}")
    v = 4
    d3 = to_dev(t3)
    fn = bc.lib.bc_ccsdt_d1_tile if family == "d1" else bc.lib.bc_ccsdt_d2_tile
    import ctypes
    a, b = to_dev(t2s[v - 1]), to_dev(v2s[v - 1])  # keep both alive across the raw call
    st = fn(v, tile, d3.data_ptr(), a.data_ptr(), b.data_ptr(), ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert st == 0
    ref = oracle.ccsdt(family, v, ext, t3, t2s[v - 1], v2s[v - 1])
    S = oracle.ccsdt_abs_bound(family, ext, t3, [t2s[v - 1] if u == v else None for u in range(1, 10)], v2s)
    assert_abs_close(to_host(d3), ref, S, 1e-12, f"{family}_{v} tile {tile}")


def test_energy_check(bc):
    ext = (7, 6, 5, 4, 3, 9, 1)
    t3 = syn.tensor(10, (n3(ext),))
    eh = syn.tensor(60, (sum(ext[:3]),), kind=syn.KIND_RANGE, lo=-2.0, hi=-0.5)
    ep = syn.tensor(61, (sum(ext[3:6]),), kind=syn.KIND_RANGE, lo=0.5, hi=2.0)
    got = float(bc.check_energy(ext, to_dev(t3), to_dev(eh), to_dev(ep)).item())
    ref = oracle.energy(ext, t3, eh, ep)
    assert abs(got - ref) <= 1e-12 * abs(ref)


@pytest.mark.parametrize("family", ["d1", "d2"])
@pytest.mark.parametrize("ext", [(16,) * 7, (32, 32, 32, 2, 2, 2, 16), (20, 20, 20, 3, 3, 3, 12)])
def test_fused_energy(bc, family, ext):
    """bc_ccsdt_fused_energy: t3 += the fused family, ws[0] = energy check of the updated
    t3.  Full 16-cubes take the energy fused into the tensor-core kernel's store pass
    (tile 16; 32^3 holes = 8 cubes per plane); 20^3 holes (ragged cubes) run the separate
    pass.  t3 bitwise equal to bc_ccsdt_*_fused; the energy equal to the oracle's energy of
    the oracle-updated t3 within 1e-12 relative (the oracle: R18 definition)."""
    na, nb = sizes(family, ext)
    t3 = syn.tensor(10, (n3(ext),))
    t2s = [syn.tensor(20 + v, (na,)) for v in range(1, 10)]
    v2s = [syn.tensor(40 + v, (nb,)) for v in range(1, 10)]
    eh = syn.tensor(60, (sum(ext[:3]),), kind=syn.KIND_RANGE, lo=-2.0, hi=-0.5)
    ep = syn.tensor(61, (sum(ext[3:6]),), kind=syn.KIND_RANGE, lo=0.5, hi=2.0)
    dt2, dv2 = [to_dev(x) for x in t2s], [to_dev(x) for x in v2s]
    a3, b3 = to_dev(t3), to_dev(t3)
    ws = torch.full((bc.BC_CHECK_WS_DOUBLES,), float("nan"), dtype=torch.float64, device="cuda")
    bc.ccsdt_fused(family, ext, a3, dt2, dv2)
    got = float(bc.ccsdt_fused_energy(family, ext, b3, dt2, dv2, to_dev(eh), to_dev(ep), ws).item())
    assert torch.equal(a3, b3)
    sep = float(bc.check_energy(ext, a3, to_dev(eh), to_dev(ep)).item())
    ref_t3 = oracle.ccsdt_fused(family, ext, t3, t2s, v2s)
    ref = oracle.energy(ext, ref_t3, eh, ep)
    assert abs(got - ref) <= 1e-12 * abs(ref), (got, ref)
    assert abs(got - sep) <= 1e-12 * abs(ref)


# (24, ...) takes the exact-24-cube kernel (ccsdt_triples24_kernel): k = 8 (one chunk) and
# k = 10 (a ragged second chunk, zero-filled by TMA)
@pytest.mark.parametrize("ext", [(16,) * 7, (20, 20, 20, 4, 4, 4, 6), (24, 24, 24, 2, 2, 2, 8), (24, 24, 24, 2, 2, 2, 10)])
@pytest.mark.parametrize("mask", ["all", "some"])
def test_triples_energy_f4(bc, ext, mask):
    """f4: all 27 variants fused, t3 never stored, energy epilogue == oracle energy of the t3
    built by the 27 per-variant oracle calls on a zeroed buffer.  Bound: |dE| <=
    sum 2|t3| dt3 / |den| with dt3 = 1e-12 * S (R14) plus the summation rounding of E."""
    H, P = ext[0], ext[3]
    fams = {}
    for fam, base in (("s1", 50), ("d1", 20), ("d2", 20 + 200000)):
        na, nb = sizes(fam, ext)
        xs = [syn.tensor(base + v, (na,)) for v in range(1, 10)]
        ys = [syn.tensor(base + 20 + v, (nb,)) for v in range(1, 10)]
        if mask == "some":
            keep = {"s1": (1, 4), "d1": (2, 5, 9), "d2": (1, 6, 7, 8)}[fam]
            xs = [x if v in keep else None for v, x in enumerate(xs, 1)]
        fams[fam] = (xs, ys)
    eh = syn.tensor(60, (3 * H,), kind=syn.KIND_RANGE, lo=-2.0, hi=-0.5)
    ep = syn.tensor(61, (3 * P,), kind=syn.KIND_RANGE, lo=0.5, hi=2.0)
    t3 = np.zeros(n3(ext))
    S = np.zeros(n3(ext))
    for fam in ("s1", "d1", "d2"):
        xs, ys = fams[fam]
        t3 = oracle.ccsdt_fused(fam, ext, t3, xs, ys)
        S += oracle.ccsdt_abs_bound(fam, ext, np.zeros(n3(ext)), xs, ys)
    E = oracle.energy(ext, t3, eh, ep)
    # per-element bound: 2 |t3| * 1e-12 S / |den|; computed with the oracle's energy on |t3|*S
    bound_t = 2.0 * 1e-12 * abs(oracle.energy(ext, np.sqrt(np.abs(t3) * S), eh, ep))
    tol = bound_t + 1e-14 * abs(E) + 1e-300
    dv = lambda xs: [None if x is None else to_dev(x) for x in xs]
    got = bc.ccsdt_triples_energy(ext, *((dv(fams[f][0]), dv(fams[f][1])) for f in ("s1", "d1", "d2")),
                                  to_dev(eh), to_dev(ep)).item()
    assert abs(got - E) <= tol, (got, E, tol)


@pytest.mark.parametrize("family", ["d1", "d2"])
@pytest.mark.parametrize("ext", [(16, 16, 16, 3, 3, 3, 8), (20, 20, 20, 4, 4, 4, 6)])
def test_tma_short_classes_no_flush_race(bc, family, ext):
    """Regression: on the warp-specialised TMA path consumer warps meet only at unit
    boundaries; with one k-chunk and one entry per class a fast warp used to flush the next
    class onto cube positions a slow warp was still updating (lost updates).  Integer data,
    bitwise, repeated."""
    na, nb = sizes(family, ext)
    t3 = syn.tensor(10, (n3(ext),), kind=syn.KIND_INT)
    t2s = [syn.tensor(20 + v, (na,), kind=syn.KIND_INT) for v in range(1, 10)]
    v2s = [syn.tensor(40 + v, (nb,), kind=syn.KIND_INT) for v in range(1, 10)]
    for mask in ((1, 2, 3), (1, 5, 9), tuple(range(1, 10))):
        a = [t2s[v - 1] if v in mask else None for v in range(1, 10)]
        ref = oracle.ccsdt_fused(family, ext, t3, a, v2s)
        for _ in range(3):
            d3 = to_dev(t3)
            bc.ccsdt_fused(family, ext, d3, [None if x is None else to_dev(x) for x in a], [to_dev(x) for x in v2s])
            assert np.array_equal(to_host(d3), ref), f"{family} {ext} mask={mask}"
