"""Algorithmic work accounting for the hot path.

Plain arithmetic on sizes only: no torch, no product library, no oracle.  Both the bench's
GPU arm (through the product's `workload` module) and its oracle legs (cpu_baseline,
--impl reference) import it, so the reference arm never loads libbarracuda.so.

Only the work the method must do is counted (the factored counts, never the naive
O(P1^6) nest); bytes are the compulsory HBM traffic: every input read once, every output
written once (operators of 8 P1^2 bytes are negligible and not counted).
"""
from __future__ import annotations

from dataclasses import dataclass

METRIC = "fp64 GFLOP/s & % of HBM/FP64 roofline for batched small contractions, 1-8 GPU"


@dataclass
class StepConfig:
    """One bench step.  n_elem / blocks are per GPU ("weak") or global
    ("strong", sharded over the ranks)."""
    p: int = 12
    n_elem: int = 262144
    tile: int = 16
    blocks: int = 8
    families: tuple = ("d1", "d2")

    @property
    def P1(self) -> int:
        return self.p + 1


# ---------------------------------------------------------------- per unit (flops, bytes)
def sumfact3d(P1: int, n: int = 1, check: bool = False):
    """V = (C x B x A) U per element: 3 stages x 2 P1^4 flops; U in, V out."""
    return 6.0 * P1 ** 4 * n + (2.0 * P1 ** 3 * n if check else 0.0), 16.0 * P1 ** 3 * n


def sumfact2d(P1: int, n: int = 1):
    """V = B U A^T per element: 2 stages x 2 P1^3 flops."""
    return 4.0 * P1 ** 3 * n, 16.0 * P1 ** 2 * n


def local_grad3(P1: int, n: int = 1):
    """ur, us, ut: 3 x 2 P1^4 flops; U in, three fields out."""
    return 6.0 * P1 ** 4 * n, 32.0 * P1 ** 3 * n


def local_grad3_t(P1: int, n: int = 1):
    """u = sum of D^T along each axis of ur/us/ut: 3 x 2 P1^4 + 2 P1^3 flops; 3 in, 1 out."""
    return 6.0 * P1 ** 4 * n + 2.0 * P1 ** 3 * n, 32.0 * P1 ** 3 * n


def ax_e(P1: int, n: int = 1):
    """Lg3 + 6-factor geometric mix + Lg3t: 12 P1^4 + 17 P1^3 flops; U, G(6), W."""
    return (12.0 * P1 ** 4 + 17.0 * P1 ** 3) * n, 64.0 * P1 ** 3 * n


def ccsdt_variants(ext, nvar: int, family: str = "d1"):
    """nvar d1/d2 variants on one t3 (read + written once): 2 |t3| k flops per variant;
    bytes 16 |t3| + 8 (|t2| + |v2|) per variant.  s1: 2 |t3| flops, operands t1 + v2."""
    h1, h2, h3, p4, p5, p6, k = ext
    n3 = h1 * h2 * h3 * p4 * p5 * p6
    if family == "s1":
        return 2.0 * n3 * nvar, 16.0 * n3 + 8.0 * nvar * (p4 * h1 + h3 * h2 * p6 * p5)
    if family == "d1":
        nop = k * p4 * p5 * h1 + h3 * h2 * p6 * k
    else:
        nop = k * p4 * h1 * h2 + k * h3 * p6 * p5
    return 2.0 * n3 * k * nvar, 16.0 * n3 + 8.0 * nvar * nop


def triples_energy(ext):
    """f4: all 27 triples variants (9 s1 + 9 d1 + 9 d2) into a t3 that is never stored,
    plus the energy epilogue (~4 flops per element beyond the sums); bytes = the operands
    (t3 neither read nor written)."""
    h1, h2, h3, p4, p5, p6, k = ext
    n3 = h1 * h2 * h3 * p4 * p5 * p6
    fl = ccsdt_variants(ext, 9, "d1")[0] + ccsdt_variants(ext, 9, "d2")[0] + ccsdt_variants(ext, 9, "s1")[0]
    ops = 9 * ((p4 * h1 + h3 * h2 * p6 * p5) + (k * p4 * p5 * h1 + h3 * h2 * p6 * k) +
               (k * p4 * h1 * h2 + k * h3 * p6 * p5))
    return fl + 4.0 * n3, 8.0 * ops


def energy(ext):
    """Energy-style check over one t3: ~9 flops per element (denominator + t^2/den)."""
    n3 = 1
    for x in ext[:6]:
        n3 *= x
    return 9.0 * n3, 8.0 * n3


# ---------------------------------------------------------------- the bench step
def flops_bytes(cfg: StepConfig, n_elem: int | None = None) -> dict:
    """(flops, bytes) per launch of every kernel of the step, for n_elem elements (default
    cfg.n_elem) and one CCSD(T) block."""
    P1 = cfg.P1
    N = cfg.n_elem if n_elem is None else n_elem
    ext = (cfg.tile,) * 7
    out = {
        "local_grad3": local_grad3(P1, N),
        "sumfact3d": sumfact3d(P1, N, check=True),  # + fused sum V^2
        "sumfact2d": sumfact2d(P1, N * P1),          # the same memory as N*P1 2-D elements
    }
    for fam in cfg.families:
        out[f"ccsdt_{fam}_fused"] = ccsdt_variants(ext, 9, fam)
    out["check_energy"] = energy(ext)
    return out


def step_flops(cfg: StepConfig, n_elem: int, blocks: int) -> float:
    """Algorithmic flops of one step over n_elem elements and `blocks` CCSD(T) blocks
    (check scalars not counted)."""
    fb = flops_bytes(cfg, n_elem)
    tot = fb["local_grad3"][0] + fb["sumfact3d"][0] + fb["sumfact2d"][0]
    tot += sum(fb[f"ccsdt_{f}_fused"][0] for f in cfg.families) * blocks
    return tot
