"""Pins of the CCSD(T) oracle (CPU only): reshaped numpy.matmul GEMM (bitwise on
integers, unequal extents), one-hot bookkeeping, sign = antisymmetriser parity,
accumulate semantics, fused = sequential, check scalars by brute force."""
import itertools
import math

import numpy as np
import pytest

import oracle
import synthetic as syn

EXT = (3, 4, 5, 6, 2, 7, 3)  # (h1, h2, h3, p4, p5, p6, k): all distinct -> swaps are caught
NAME_IDX = {n: i for i, n in enumerate(oracle.NAMES)}


def shapes(family, ext):
    h1, h2, h3, p4, p5, p6, k = ext
    if family == "d1":
        return (k, p4, p5, h1), (h3, h2, p6, k)        # t2[h7,p4,p5,h1], v2[h3,h2,p6,h7]
    if family == "d2":
        return (k, p4, h1, h2), (k, h3, p6, p5)        # t2[p7,p4,h1,h2], v2[p7,h3,p6,p5]
    return (p4, h1), (h3, h2, p6, p5)                  # t1[p4,h1],       v2[h3,h2,p6,p5]


def fortran(shape, tid, kind=syn.KIND_INT):
    """Flat array holding a Fortran-ordered tensor of `shape` (values by flat position)."""
    return syn.tensor(tid, (int(np.prod(shape)),), kind=kind)


def as_named(flat, shape):
    return flat.reshape(shape, order="F")


def contraction_by_matmul(family, ext, t2, v2):
    """X[h1,h2,h3,p4,p5,p6] (named axes, in NAMES order) via reshaped GEMM."""
    h1, h2, h3, p4, p5, p6, k = ext
    s2, sv = shapes(family, ext)
    T, V = as_named(t2, s2), as_named(v2, sv)
    if family == "d1":
        Tm = T.reshape(k, p4 * p5 * h1, order="F")                 # [h7] x [(p4,p5,h1)]
        Vm = np.moveaxis(V, 3, 0).reshape(k, h3 * h2 * p6, order="F")  # [h7] x [(h3,h2,p6)]
        X = (Vm.T @ Tm).reshape(h3, h2, p6, p4, p5, h1, order="F")
        return X.transpose(5, 1, 0, 3, 4, 2)  # -> h1,h2,h3,p4,p5,p6
    if family == "d2":
        Tm = T.reshape(k, p4 * h1 * h2, order="F")                 # [p7] x [(p4,h1,h2)]
        Vm = V.reshape(k, h3 * p6 * p5, order="F")                 # [p7] x [(h3,p6,p5)]
        X = (Vm.T @ Tm).reshape(h3, p6, p5, p4, h1, h2, order="F")
        return X.transpose(4, 5, 0, 3, 2, 1)
    X = np.einsum("ad,bcef->dcbaef", T, V)  # outer product: t1[p4,h1] v2[h3,h2,p6,p5]
    # dims now (h1, h2, h3, p4, p6, p5) -> swap last two
    return X.transpose(0, 1, 2, 3, 5, 4)


def store(X_named, order, ext):
    """Flatten named tensor X into the Fortran layout whose position q holds order[q]."""
    perm = [NAME_IDX[n] for n in order]
    return X_named.transpose(perm).ravel(order="F")


def perm_parity(seq, ref):
    p = [ref.index(s) for s in seq]
    par = 1
    for i in range(len(p)):
        for j in range(i + 1, len(p)):
            if p[i] > p[j]:
                par = -par
    return par


@pytest.mark.parametrize("family", ["d1", "d2", "s1"])
@pytest.mark.parametrize("variant", range(1, 10))
def test_ccsdt_matches_reshaped_gemm_bitwise(family, variant):
    s2, sv = shapes(family, EXT)
    t2, v2 = fortran(s2, 20 + variant), fortran(sv, 40 + variant)
    t3 = fortran((int(np.prod(EXT[:6])),), 10)
    order, sign = oracle.variant_table(family, variant)
    ref = t3 + sign * store(contraction_by_matmul(family, EXT, t2, v2), order, EXT)
    got = oracle.ccsdt(family, variant, EXT, t3, t2, v2)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("family", ["d1", "d2", "s1"])
def test_variant_table_rules(family):
    """Sign = -(hole parity)(particle parity) for d1/d2 and + for s1 (antisymmetriser
    P(i/jk)P(a/bc)); hole permutation cycles fastest in v, particle permutation slowest;
    generating rule of DESIGN.md reading R12."""
    holes0, parts0 = ("h3", "h2", "h1"), ("p6", "p5", "p4")
    seen = set()
    for v in range(1, 10):
        order, sign = oracle.variant_table(family, v)
        hol, par = order[:3], order[3:]
        assert sorted(hol) == sorted(holes0) and sorted(par) == sorted(parts0)
        base = -1 if family in ("d1", "d2") else 1
        assert sign == base * perm_parity(hol, holes0) * perm_parity(par, parts0)
        seen.add(order)
        o1, _ = oracle.variant_table(family, 1 + (v - 1) % 3)
        o2, _ = oracle.variant_table(family, 1 + 3 * ((v - 1) // 3))
        assert hol == o1[:3] and par == o2[3:]
        i = (v - 1) % 3
        j = (v - 1) // 3
        if family in ("d1", "s1"):
            assert hol.index("h1") == 2 - i and [h for h in hol if h != "h1"] == ["h3", "h2"]
        else:
            assert hol.index("h3") == [0, 2, 1][i] and [h for h in hol if h != "h3"] == ["h2", "h1"]
        if family == "d1":
            assert par.index("p6") == [0, 2, 1][j] and [q for q in par if q != "p6"] == ["p5", "p4"]
        else:
            assert par.index("p4") == 2 - j and [q for q in par if q != "p4"] == ["p6", "p5"]
    assert len(seen) == 9


@pytest.mark.parametrize("family", ["d1", "d2"])
@pytest.mark.parametrize("variant", [1, 5, 9])
def test_ccsdt_one_hot_bookkeeping(family, variant):
    """A one-hot t2 changes t3 exactly at the positions the contraction touches, by
    s_v * v2(..., k*)."""
    h1, h2, h3, p4, p5, p6, k = EXT
    s2, sv = shapes(family, EXT)
    v2 = fortran(sv, 41)
    T = np.zeros(s2, order="F")
    if family == "d1":
        star = dict(k=1, p4=3, p5=1, h1=2)
        T[star["k"], star["p4"], star["p5"], star["h1"]] = 1.0
    else:
        star = dict(k=2, p4=4, h1=1, h2=3)
        T[star["k"], star["p4"], star["h1"], star["h2"]] = 1.0
    t2 = T.ravel(order="F")
    t3 = np.zeros(int(np.prod(EXT[:6])))
    out = oracle.ccsdt(family, variant, EXT, t3, t2, v2)
    order, sign = oracle.variant_table(family, variant)
    V = as_named(v2, sv)
    X = np.zeros((h1, h2, h3, p4, p5, p6))
    for a, b, c, d, e, f in itertools.product(range(h1), range(h2), range(h3), range(p4), range(p5), range(p6)):
        if family == "d1" and (a, d, e) == (star["h1"], star["p4"], star["p5"]):
            X[a, b, c, d, e, f] = V[c, b, f, star["k"]]
        if family == "d2" and (a, b, d) == (star["h1"], star["h2"], star["p4"]):
            X[a, b, c, d, e, f] = V[star["k"], c, f, e]
    assert np.array_equal(out, sign * store(X, order, EXT))


def test_ccsdt_accumulate_and_fused_equals_sequential():
    s2, sv = shapes("d2", EXT)
    t3 = fortran((int(np.prod(EXT[:6])),), 10)
    t2s = [fortran(s2, 20 + v) for v in range(1, 10)]
    v2s = [fortran(sv, 40 + v) for v in range(1, 10)]
    seq = t3.copy()
    for v in range(1, 10):
        contrib = oracle.ccsdt("d2", v, EXT, np.zeros_like(t3), t2s[v - 1], v2s[v - 1])
        seq = seq + contrib
    fused = oracle.ccsdt_fused("d2", EXT, t3, t2s, v2s)
    assert np.array_equal(fused, seq)  # integers: exact
    mask = [t if v % 2 else None for v, t in enumerate(t2s, 1)]
    part = oracle.ccsdt_fused("d2", EXT, t3, mask, v2s)
    ref = t3.copy()
    for v in (1, 3, 5, 7, 9):
        ref = oracle.ccsdt("d2", v, EXT, ref, t2s[v - 1], v2s[v - 1])
    assert np.array_equal(part, ref)


def test_sumsq_and_energy_brute_force():
    x = syn.tensor(1, (1001,))
    assert abs(oracle.sumsq(x) - math.fsum(x * x)) <= 1e-13 * math.fsum(x * x)
    ext = (2, 3, 2, 3, 2, 2, 1)
    h1, h2, h3, p4, p5, p6, _ = ext
    n = h1 * h2 * h3 * p4 * p5 * p6
    t3 = syn.tensor(10, (n,))
    eh = syn.tensor(60, (h1 + h2 + h3,), kind=syn.KIND_RANGE, lo=-2.0, hi=-0.5)
    ep = syn.tensor(61, (p4 + p5 + p6,), kind=syn.KIND_RANGE, lo=0.5, hi=2.0)
    T = t3.reshape((h3, h2, h1, p6, p5, p4), order="F")
    terms = []
    for c, b, a, f, e, d in itertools.product(range(h3), range(h2), range(h1), range(p6), range(p5), range(p4)):
        den = eh[h1 + h2 + c] + eh[h1 + b] + eh[a] - ep[p4 + p5 + f] - ep[p4 + e] - ep[d]
        terms.append(T[c, b, a, f, e, d] ** 2 / den)
    E = oracle.energy(ext, t3, eh, ep)
    assert E < 0 and abs(E - math.fsum(terms)) <= 1e-13 * abs(math.fsum(terms))
