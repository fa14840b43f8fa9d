"""The bench "step": one pass of every hot-path row of SURVEY §8(a) over one batch of
synthetic input resident in HBM.

Per GPU (weak scaling: every rank owns its own slice of the global batch):
  a6-a8  local_grad3  p=12, N elements      (BASELINE configs[1]: p=12, N=262,144)
  a1-a4  sumfact3d    p=12, the SAME N elements (fused S1-S3)
  a5     sumfact2d    p=12, the same memory viewed as N*(p+1) 2-D elements
  a9-a11 CCSD(T) d1 and d2, 9 variants each, fused, tile 16 (configs[2], configs[3]),
         `blocks` tile blocks, each with its own t3 / t2_v / v2_v
  a12    check scalars: sum V^2 and the energy-style sum of every t3, then SUM over ranks
Inputs are generated on the device by the counter-based generator keyed by GLOBAL
indices (element e of rank r is global element r*N + e), so any element or block can be
regenerated on the host by `synthetic` for verification.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

import synthetic as syn

from . import ccsdt_fused, check_energy, fill, local_grad3, sumfact2d, sumfact3d
from . import dist as bdist


@dataclass
class StepConfig:
    p: int = 12
    n_elem: int = 262144          # per GPU
    tile: int = 16
    blocks: int = 8               # CCSD(T) tile blocks per GPU
    families: tuple = ("d1", "d2")

    @property
    def P1(self) -> int:
        return self.p + 1


def flops_bytes(cfg: StepConfig) -> dict:
    """Algorithmic flops and HBM bytes per kernel launch."""
    P1, N, t = cfg.P1, cfg.n_elem, cfg.tile
    n3 = t ** 6
    nop = t ** 4
    out = {
        "local_grad3": (6.0 * P1 ** 4 * N, 32.0 * P1 ** 3 * N),
        "sumfact3d": (6.0 * P1 ** 4 * N + 2.0 * P1 ** 3 * N, 16.0 * P1 ** 3 * N),  # + fused sum V^2
        "sumfact2d": (4.0 * P1 ** 3 * (N * P1), 16.0 * P1 ** 2 * (N * P1)),
    }
    for fam in cfg.families:
        out[f"ccsdt_{fam}_fused"] = (9 * 2.0 * n3 * t, 16.0 * n3 + 9 * 8.0 * 2 * nop)
    out["check_energy"] = (9.0 * n3, 8.0 * n3)
    return out


@dataclass
class Step:
    cfg: StepConfig
    rank: int = 0
    world: int = 1
    device: torch.device = field(default_factory=lambda: torch.device("cuda"))

    def __post_init__(self):
        c, dev, f64 = self.cfg, self.device, torch.float64
        P1, N = c.P1, c.n_elem
        self.e0 = self.rank * N                      # global element offset of this rank
        self.b0 = self.rank * c.blocks               # global CCSD(T) block offset
        npts = P1 ** 3
        self.U = torch.empty((N, P1, P1, P1), dtype=f64, device=dev)
        fill(self.U, syn.TID["U"], offset=self.e0 * npts)
        self.A, self.B, self.C = (torch.empty((P1, P1), dtype=f64, device=dev) for _ in range(3))
        for t, name in ((self.A, "A"), (self.B, "B"), (self.C, "C")):
            fill(t, syn.TID[name])
        self.D = torch.from_numpy(syn.gll_derivative(c.p)).to(dev)
        self.V = torch.empty_like(self.U)
        self.ur, self.us, self.ut = (torch.empty_like(self.U) for _ in range(3))
        self.U2 = self.U.view(N * P1, P1, P1)          # the same batch as 2-D elements
        self.V2 = torch.empty_like(self.U2)
        t = c.tile
        self.ext = (t,) * 7
        self.t3, self.t2, self.v2 = [], {}, {}
        for b in range(c.blocks):
            gb = self.b0 + b
            t3 = torch.empty(t ** 6, dtype=f64, device=dev)
            fill(t3, syn.ccsdt_block_tid(syn.TID["T3"], 0, gb))
            self.t3.append(t3)
            for fam in c.families:
                base = 0 if fam == "d1" else 200000  # d2 operands get their own ids
                self.t2[(fam, b)] = [fill(torch.empty(t ** 4, dtype=f64, device=dev),
                                          syn.ccsdt_block_tid(syn.TID["T2"] + base, v, gb)) for v in range(1, 10)]
                self.v2[(fam, b)] = [fill(torch.empty(t ** 4, dtype=f64, device=dev),
                                          syn.ccsdt_block_tid(syn.TID["V2"] + base, v, gb)) for v in range(1, 10)]
        self.eps_h = fill(torch.empty(3 * t, dtype=f64, device=dev), syn.TID["EPS_H"], kind=syn.KIND_RANGE,
                          lo=-2.0, hi=-0.5)
        self.eps_p = fill(torch.empty(3 * t, dtype=f64, device=dev), syn.TID["EPS_P"], kind=syn.KIND_RANGE,
                          lo=0.5, hi=2.0)
        self.ws = torch.zeros((1 + c.blocks, 1024), dtype=f64, device=dev)
        self.checks = torch.zeros(2, dtype=f64, device=dev)
        self.fb = flops_bytes(c)

    # ------------------------------------------------------------------------------
    def inputs(self):
        """Tensors a host-fed (e2e) step must copy in before computing."""
        ins = [self.U, self.A, self.B, self.C, self.D, self.eps_h, self.eps_p] + self.t3
        for key in sorted(self.t2):
            ins += self.t2[key] + self.v2[key]
        return ins

    def run(self, timer=None) -> torch.Tensor:
        """One step.  `timer(name)` (optional) is called after each launch group."""
        c = self.cfg
        tick = timer or (lambda name: None)
        local_grad3(self.D, self.U, out=(self.ur, self.us, self.ut))
        tick("local_grad3")
        sumfact3d(self.A, self.B, self.C, self.U, out=self.V, check_ws=self.ws[0])  # + fused sum V^2
        tick("sumfact3d")
        sumfact2d(self.A, self.B, self.U2, out=self.V2)
        tick("sumfact2d")
        for fam in c.families:
            for b in range(c.blocks):
                ccsdt_fused(fam, self.ext, self.t3[b], self.t2[(fam, b)], self.v2[(fam, b)])
            tick(f"ccsdt_{fam}_fused")
        for b in range(c.blocks):
            check_energy(self.ext, self.t3[b], self.eps_h, self.eps_p, self.ws[1 + b])
        tick("check_energy")
        self.checks[0] = self.ws[0, 0]
        self.checks[1] = self.ws[1:, 0].sum()
        bdist.all_reduce_sum_(self.checks)
        return self.checks

    def launches_per_step(self) -> dict:
        c = self.cfg
        return {"local_grad3": 1, "sumfact3d": 1, "sumfact2d": 1,
                **{f"ccsdt_{f}_fused": c.blocks for f in c.families},
                "check_energy": 2 * c.blocks}

    def flops_per_step(self) -> float:
        c = self.cfg
        tot = 0.0
        for k, n in self.launches_per_step().items():
            if k.startswith("check"):
                continue
            tot += self.fb[k][0] * (1 if not k.startswith("ccsdt") else c.blocks)
        return tot

    # ------------------------------------------------------------------------------
    def sample_elements(self, n: int, seed: int = 0) -> np.ndarray:
        """Local element ids to verify: first, last and a seeded sample (DESIGN R21)."""
        N = self.cfg.n_elem
        rng = np.random.default_rng(1234 + seed + self.rank)
        s = set(rng.choice(N, size=min(n, N), replace=False).tolist()) | {0, N - 1}
        return np.array(sorted(s), dtype=np.int64)
