"""The bench "step": one pass of every hot-path row of SURVEY §8(a) over one batch of
synthetic input resident in HBM, and its copy-inclusive form.

Per rank:
  a6-a8  local_grad3  p=12 on the rank's elements (BASELINE configs[1]: p=12, N=262,144)
  a1-a4  sumfact3d    p=12 on the SAME elements (fused S1-S3, fused sum V^2)
  a5     sumfact2d    p=12, the same memory viewed as n*(p+1) 2-D elements
  a9-a11 CCSD(T) d1 and d2, 9 variants each, fused, tile 16 (configs[2], configs[3]) on the
         rank's tile blocks, each with its own t3 / t2_v / v2_v
  a12    check scalars: sum V^2 and the energy-style sum of every t3, then SUM over ranks
Sharding (units are independent):
  weak   rank r owns global elements [r N, (r+1) N) and blocks [r B, (r+1) B)
  strong the global batch (N elements, B blocks) is split by dist.shard(): rank r owns
         [floor(r N / G), floor((r+1) N / G)) and likewise for blocks
Inputs are generated on the device by the counter-based generator keyed by GLOBAL
indices, so an element's or block's values, and therefore its outputs, do not depend on
G or on the sharding mode (tested bitwise, tests/test_scaling_invariance.py), and any
element or block can be regenerated on the host by `synthetic` for verification.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

import accounting
import synthetic as syn
from accounting import StepConfig  # noqa: F401  (re-export)

from . import ccsdt_fused, ccsdt_fused_energy, check_energy, fill, local_grad3, sumfact2d, sumfact3d
from . import dist as bdist


@dataclass
class Step:
    cfg: StepConfig
    rank: int = 0
    world: int = 1
    device: torch.device = field(default_factory=lambda: torch.device("cuda"))
    scaling: str = "weak"

    def __post_init__(self):
        c, dev, f64 = self.cfg, self.device, torch.float64
        if self.scaling == "weak":
            self.e0, self.n = self.rank * c.n_elem, c.n_elem
            self.b0, self.nb = self.rank * c.blocks, c.blocks
        elif self.scaling == "strong":
            a, b = bdist.shard(c.n_elem, self.rank, self.world)
            self.e0, self.n = a, b - a
            a, b = bdist.shard(c.blocks, self.rank, self.world)
            self.b0, self.nb = a, b - a
        else:
            raise ValueError("scaling must be 'weak' or 'strong'")
        P1, N = c.P1, self.n
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
        for b in range(self.nb):
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
        self.ws = torch.zeros((1 + max(self.nb, 1), 1024), dtype=f64, device=dev)
        self.checks = torch.zeros(2, dtype=f64, device=dev)
        self.fb = accounting.flops_bytes(c, self.n)

    # ------------------------------------------------------------------------------
    def inputs(self):
        """Tensors a host-fed (e2e) step must copy in before computing."""
        ins = [self.U, self.A, self.B, self.C, self.D, self.eps_h, self.eps_p] + self.t3
        for key in sorted(self.t2):
            ins += self.t2[key] + self.v2[key]
        return ins

    def outputs(self):
        """Every result of the step: the spectral fields and the updated t3 blocks."""
        return [self.ur, self.us, self.ut, self.V, self.V2] + self.t3

    def run(self, timer=None) -> torch.Tensor:
        """One step.  `timer(name)` (optional) is called after each launch group."""
        c = self.cfg
        tick = timer or (lambda name: None)
        if self.n:
            local_grad3(self.D, self.U, out=(self.ur, self.us, self.ut))
            tick("local_grad3")
            sumfact3d(self.A, self.B, self.C, self.U, out=self.V, check_ws=self.ws[0])  # + fused sum V^2
            tick("sumfact3d")
            sumfact2d(self.A, self.B, self.U2, out=self.V2)
            tick("sumfact2d")
        else:
            self.ws[0, 0] = 0.0
        # the energy check scalar of each block rides in the last family's call (fused into
        # its t3 store pass, bc_ccsdt_fused_energy)
        for i, fam in enumerate(c.families):
            last = i + 1 == len(c.families)
            for b in range(self.nb):
                if last:
                    ccsdt_fused_energy(fam, self.ext, self.t3[b], self.t2[(fam, b)], self.v2[(fam, b)],
                                       self.eps_h, self.eps_p, self.ws[1 + b])
                else:
                    ccsdt_fused(fam, self.ext, self.t3[b], self.t2[(fam, b)], self.v2[(fam, b)])
            tick(f"ccsdt_{fam}_fused")
        if not c.families:
            for b in range(self.nb):
                check_energy(self.ext, self.t3[b], self.eps_h, self.eps_p, self.ws[1 + b])
            tick("check_energy")
        self.checks[0] = self.ws[0, 0]
        self.checks[1] = self.ws[1:1 + self.nb, 0].sum()
        bdist.all_reduce_sum_(self.checks)
        return self.checks

    def launches_per_step(self) -> dict:
        c = self.cfg
        return {"local_grad3": 1, "sumfact3d": 1, "sumfact2d": 1,
                **{f"ccsdt_{f}_fused": self.nb for f in c.families},
                **({} if c.families else {"check_energy": 2 * self.nb})}

    def flops_per_step(self) -> float:
        """Algorithmic flops of this rank's share of the step."""
        return accounting.step_flops(self.cfg, self.n, self.nb)

    # ------------------------------------------------------------------------------
    def sample_elements(self, n: int, seed: int = 0) -> np.ndarray:
        """Local element ids to verify: first, last and a seeded sample (DESIGN R21)."""
        N = self.n
        rng = np.random.default_rng(1234 + seed + self.rank)
        s = set(rng.choice(N, size=min(n, N), replace=False).tolist()) | {0, N - 1}
        return np.array(sorted(s), dtype=np.int64)


class HostPipeline:
    """The step fed from and returned to pinned host memory (the e2e measurement,
    DESIGN.md §5; the paper's timings include both copy directions).

    The spectral batch is cut into `chunks` contiguous element ranges and every CCSD(T)
    block is its own chunk.  Three streams overlap the work: H2D copies of chunk i+1 and
    D2H copies of chunk i-1 run while chunk i computes, so a step costs about
    max(H2D bytes / H2D bandwidth, D2H bytes / D2H bandwidth) instead of their sum plus
    the compute.  Events order each chunk's copy-in -> compute -> copy-out, and across
    steps the next copy-in of a buffer after the compute that read it / the copy-out that
    read its result.  Every output (ur, us, ut, V, V2, all t3 blocks) and the two check
    scalars reach the host every step (outputs into a ring of pinned slots, see below)."""

    def __init__(self, step: Step, chunks: int = 16, out_slots: int = 2):
        self.st = step
        dev = step.device
        n = step.n
        self.bounds = [(n * i // chunks, n * (i + 1) // chunks) for i in range(chunks)] if n else []
        self.bounds = [(a, b) for a, b in self.bounds if b > a]
        pin = lambda t: torch.empty(t.shape, dtype=t.dtype, pin_memory=True)  # noqa: E731
        self.h_in = {id(t): pin(t) for t in step.inputs()}
        for t in step.inputs():
            self.h_in[id(t)].copy_(t)
        # outputs land in a ring of `out_slots` pinned chunk slots per output (spectral) and
        # per-block slots (t3): every result byte crosses PCIe every step, while the pinned
        # footprint stays ~(inputs + 2 chunks) per rank (8 ranks x 30 GB of fully pinned
        # outputs would not fit the box's host memory)
        self.out_slots = out_slots
        cmax = max([b - a for a, b in self.bounds] or [0])
        P1 = step.cfg.P1
        self.h_ring = {nm: [torch.empty((cmax,) + tuple(getattr(step, nm).shape[1:]), dtype=torch.float64,
                                        pin_memory=True) for _ in range(out_slots)]
                       for nm in ("ur", "us", "ut", "V")}
        self.h_ring["V2"] = [torch.empty((cmax * P1, P1, P1), dtype=torch.float64, pin_memory=True)
                             for _ in range(out_slots)]
        self.h_t3 = [pin(step.t3[0]) for _ in range(min(out_slots, step.nb))] if step.nb else []
        self.h_chk = torch.empty(2, dtype=torch.float64, pin_memory=True)
        self.s_in, self.s_cmp, self.s_out = (torch.cuda.Stream(dev) for _ in range(3))
        nunits = len(self.bounds) + step.nb
        mk = lambda: [torch.cuda.Event() for _ in range(nunits)]  # noqa: E731
        self.ev_in, self.ev_cmp, self.ev_out = mk(), mk(), mk()
        self.started = False
        self.ws = torch.zeros((len(self.bounds) + 1, 1024), dtype=torch.float64, device=dev)
        st = step
        self.small = [st.A, st.B, st.C, st.D, st.eps_h, st.eps_p]
        self.h2d_bytes = sum(t.numel() * t.element_size() for t in st.inputs())
        self.d2h_bytes = sum(t.numel() * t.element_size() for t in st.outputs()) + 16

    def _h2d(self, dst, lo=None, hi=None):
        src = self.h_in[id(dst)]
        if lo is None:
            dst.copy_(src, non_blocking=True)
        else:
            dst[lo:hi].copy_(src[lo:hi], non_blocking=True)

    def _d2h_chunk(self, name, ci, lo, hi):
        dst = self.h_ring[name][ci % self.out_slots]
        dst[:hi - lo].copy_(getattr(self.st, name)[lo:hi], non_blocking=True)

    def run(self) -> torch.Tensor:
        st, c = self.st, self.st.cfg
        P1 = c.P1
        with torch.cuda.stream(self.s_cmp):  # operators / denominators (a few KB), in
            for t in self.small:               # order with the compute that reads them
                self._h2d(t)
        u = 0
        for ci, (a, b) in enumerate(self.bounds):
            with torch.cuda.stream(self.s_in):
                if self.started:
                    self.s_in.wait_event(self.ev_cmp[u])      # previous step's compute read U
                self._h2d(st.U, a, b)
                self.ev_in[u].record(self.s_in)
            with torch.cuda.stream(self.s_cmp):
                self.s_cmp.wait_event(self.ev_in[u])
                if self.started:
                    self.s_cmp.wait_event(self.ev_out[u])     # previous step's results left
                local_grad3(st.D, st.U[a:b], out=(st.ur[a:b], st.us[a:b], st.ut[a:b]))
                sumfact3d(st.A, st.B, st.C, st.U[a:b], out=st.V[a:b], check_ws=self.ws[ci])
                sumfact2d(st.A, st.B, st.U2[a * P1:b * P1], out=st.V2[a * P1:b * P1])
                self.ev_cmp[u].record(self.s_cmp)
            with torch.cuda.stream(self.s_out):
                self.s_out.wait_event(self.ev_cmp[u])
                for nm in ("ur", "us", "ut", "V"):
                    self._d2h_chunk(nm, ci, a, b)
                self._d2h_chunk("V2", ci, a * P1, b * P1)
                self.ev_out[u].record(self.s_out)
            u += 1
        for b in range(st.nb):
            ops = [x for fam in c.families for x in st.t2[(fam, b)] + st.v2[(fam, b)]]
            with torch.cuda.stream(self.s_in):
                if self.started:
                    self.s_in.wait_event(self.ev_out[u])      # previous step's t3 left
                self._h2d(st.t3[b])
                for x in ops:
                    self._h2d(x)
                self.ev_in[u].record(self.s_in)
            with torch.cuda.stream(self.s_cmp):
                self.s_cmp.wait_event(self.ev_in[u])
                for i, fam in enumerate(c.families):
                    if i + 1 == len(c.families):
                        ccsdt_fused_energy(fam, st.ext, st.t3[b], st.t2[(fam, b)], st.v2[(fam, b)],
                                           st.eps_h, st.eps_p, st.ws[1 + b])
                    else:
                        ccsdt_fused(fam, st.ext, st.t3[b], st.t2[(fam, b)], st.v2[(fam, b)])
                if not c.families:
                    check_energy(st.ext, st.t3[b], st.eps_h, st.eps_p, st.ws[1 + b])
                self.ev_cmp[u].record(self.s_cmp)
            with torch.cuda.stream(self.s_out):
                self.s_out.wait_event(self.ev_cmp[u])
                self.h_t3[b % len(self.h_t3)].copy_(st.t3[b], non_blocking=True)
                self.ev_out[u].record(self.s_out)
            u += 1
        with torch.cuda.stream(self.s_cmp):
            st.checks[0] = self.ws[:len(self.bounds), 0].sum()
            st.checks[1] = st.ws[1:1 + st.nb, 0].sum()
            bdist.all_reduce_sum_(st.checks)
            self.s_out.wait_stream(self.s_cmp)
        with torch.cuda.stream(self.s_out):
            self.h_chk.copy_(st.checks, non_blocking=True)
        self.started = True
        return self.h_chk

    def join(self, stream: torch.cuda.Stream) -> None:
        """Make `stream` wait for everything the pipeline has issued."""
        for s in (self.s_in, self.s_cmp, self.s_out):
            stream.wait_stream(s)

    def fork(self, stream: torch.cuda.Stream) -> None:
        """Make the pipeline's streams wait for `stream` (the timing start event)."""
        for s in (self.s_in, self.s_cmp, self.s_out):
            s.wait_stream(stream)
