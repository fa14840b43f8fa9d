"""Seeded synthetic inputs — the ONE module shared by the oracle side and the CUDA side.

It holds none of the method's arithmetic (no contraction, no reduction): only the
counter-based generator that turns (seed, tensor id, global index) into a value, the
tensor-id table, and the GLL derivative operator that Nekbone passes to local_grad3
as an *input* (DESIGN.md "Input recipe").

Generator ("Synthetic input generator"):
    z = splitmix64(seed + (tensor_id << 40) + global_index)        (mod 2^64)
    real    : x = ((z >> 11) * 2^-53) * 2 - 1      in [-1, 1)   (exact in fp64)
    integer : x = (z >> 61) - 4                     in {-4..3}   (exact in fp64)
    shifted : x = lo + (hi - lo) * ((z >> 11) * 2^-53)            (used for eps_h / eps_p)

The CUDA library implements the same generator in its own code (`bc_fill`), and a
gpu test checks that both produce bit-identical arrays.  Because a value depends on
its global index only, any shard or any sampled element can be regenerated alone.
"""
from __future__ import annotations

import numpy as np

SEED = 2015

# tensor-id table; CCSD(T) block b adds b*100 to the id.
TID = {
    "U": 1, "A": 2, "B": 3, "C": 4, "V_POISON": 5, "D": 6,
    "UR": 7, "US": 8, "UT": 9,         # inputs of local_grad3_t (f1)
    "G": 11,                            # geometric factors of ax_e (f2)
    "T3": 10, "T2": 20, "V2": 40,       # t2_v = 20+v, v2_v = 40+v
    "T1": 50,                           # singles amplitude of s1 (f3)
    "EPS_H": 60, "EPS_P": 61,
}

KIND_REAL = 0
KIND_INT = 1
KIND_RANGE = 2

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def counter_base(seed: int, tensor_id: int) -> np.uint64:
    return np.uint64((int(seed) + (int(tensor_id) << 40)) & 0xFFFFFFFFFFFFFFFF)


def raw(tensor_id: int, index: np.ndarray, seed: int = SEED) -> np.ndarray:
    idx = np.asarray(index, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return splitmix64(counter_base(seed, tensor_id) + idx)


def values(tensor_id: int, index, kind: int = KIND_REAL, seed: int = SEED,
           lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    """fp64 values of tensor `tensor_id` at global flat indices `index`."""
    z = raw(tensor_id, index, seed)
    if kind == KIND_INT:
        return (z >> np.uint64(61)).astype(np.float64) - 4.0
    u = (z >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    if kind == KIND_REAL:
        return u * 2.0 - 1.0
    return lo + (hi - lo) * u


def tensor(tensor_id: int, shape, kind: int = KIND_REAL, seed: int = SEED, offset: int = 0,
           lo: float = -1.0, hi: float = 1.0, dtype=np.float64) -> np.ndarray:
    """A whole tensor, C-contiguous, flat index = offset + position."""
    n = int(np.prod(shape)) if len(shape) else 1
    idx = np.arange(offset, offset + n, dtype=np.uint64)
    return values(tensor_id, idx, kind, seed, lo, hi).reshape(shape).astype(dtype, copy=False)


def elements(tensor_id: int, P1: int, elems, kind: int = KIND_REAL, seed: int = SEED,
             ndim: int = 3) -> np.ndarray:
    """The listed elements of a batched spectral field [N][P1]^ndim (global element ids)."""
    npts = P1 ** ndim
    elems = np.asarray(elems, dtype=np.uint64)
    idx = elems[:, None] * np.uint64(npts) + np.arange(npts, dtype=np.uint64)[None, :]
    return values(tensor_id, idx, kind, seed).reshape((len(elems),) + (P1,) * ndim)


def ccsdt_block_tid(base: int, variant: int = 0, block: int = 0) -> int:
    return base + variant + 100 * block


# ---------------------------------------------------------------------------
# GLL derivative operator (an INPUT of local_grad3: Nekbone's D, Deville et al. [9]).
# SURVEY.md §8(c) ambiguity #11: nodes {-1, roots of P_p', +1};
# D_ij = P_p(x_i) / (P_p(x_j) (x_i - x_j)) for i != j; D_ii = -sum_{j != i} D_ij.
# ---------------------------------------------------------------------------

def _legendre(p: int, x: np.ndarray) -> np.ndarray:
    x = np.asarray(x, dtype=np.float64)
    if p == 0:
        return np.ones_like(x)
    pm1, pc = np.ones_like(x), x.copy()
    for n in range(1, p):
        pm1, pc = pc, ((2 * n + 1) * x * pc - n * pm1) / (n + 1)
    return pc


def gll_nodes(p: int) -> np.ndarray:
    """p+1 Gauss-Lobatto-Legendre nodes on [-1, 1], ascending."""
    if p < 1:
        raise ValueError("p >= 1")
    P1 = p + 1
    if p == 1:
        return np.array([-1.0, 1.0])
    # interior nodes: roots of P_p'; Newton from Chebyshev-Gauss-Lobatto guesses
    x = -np.cos(np.pi * np.arange(P1) / p)
    for _ in range(100):
        # P_p'(x) via (1-x^2) P_p' = p (P_{p-1} - x P_p); Newton on q(x) = (1-x^2) P_p'(x)
        Pp = _legendre(p, x[1:-1])
        Pm = _legendre(p - 1, x[1:-1])
        xi = x[1:-1]
        q = p * (Pm - xi * Pp)
        # q'(x) = -p (p+1) P_p(x)  (Legendre ODE)
        dq = -p * (p + 1) * Pp
        dx = q / dq
        x[1:-1] = xi - dx
        if np.max(np.abs(dx)) < 1e-16:
            break
    x[0], x[-1] = -1.0, 1.0
    return np.sort(x)


def gll_derivative(p: int) -> np.ndarray:
    """(p+1)x(p+1) row-major D with D[a][b] = h_b'(x_a) (Lagrange basis on GLL nodes)."""
    x = gll_nodes(p)
    P1 = p + 1
    L = _legendre(p, x)
    D = np.zeros((P1, P1))
    for i in range(P1):
        for j in range(P1):
            if i != j:
                D[i, j] = L[i] / (L[j] * (x[i] - x[j]))
    for i in range(P1):
        D[i, i] = -np.sum(D[i, np.arange(P1) != i])
    return D
