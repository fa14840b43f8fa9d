#!/usr/bin/env python3
"""Benchmark: fp64 GFLOP/s of one pass of the whole hot path.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl barracuda|reference]
                    [--scaling weak|strong]

N > 1 is launched by the driver with torchrun (one process per GPU, NCCL).  Units are
independent: with --scaling weak (default) each rank owns its own
slice of the global batch; with --scaling strong the global batch (--n-elem elements,
--blocks CCSD(T) blocks) is split over the ranks by dist.shard().  No data-path
collective: only the check-scalar SUM, the flop SUM and the max-over-ranks of the timing
cross GPUs.  Rank 0 prints ONE JSON line.  The default workload is BASELINE.json
configs[1] (Nekbone local_grad3, p=12, N=262,144 elements) with every other §8(a) row run
over the same batch in the same step (sumfact3d, sumfact2d, CCSD(T) d1/d2 fused tile 16,
check scalars), plus per-config rows (BASELINE configs 1, 3, 4, 5) measured in the same
run after the timed step.

The oracle (oracle/) is executed only by the cpu_baseline leg and by --impl reference;
those legs import only `oracle`, `synthetic` and `accounting` (never the product
package, so libbarracuda.so is not loaded there).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import accounting as acct  # noqa: E402
from accounting import METRIC, StepConfig  # noqa: E402

FP64_NOMINAL_TFLOPS = 37.2  # 148 SMs x 64 FP64 FMA/clk x 2 x 1.965 GHz (only if the live probe fails)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (measured copy)"
    return 6650.0, "fallback 6.65 TB/s (B200_PROFILING.md)"


def load_traffic():
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f)
    return {}


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (FileNotFoundError, OSError):
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm), "gpu": self.index}


def gather_clocks(local, rank):
    """Every rank samples its own GPU; rank 0 reports the median over ranks' medians, the
    lowest max clock, the union of throttle reasons and the per-rank summaries."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return local
    allc = [None] * dist.get_world_size()
    dist.all_gather_object(allc, local)
    sm = [c["sm_mhz"] for c in allc if c.get("sm_mhz") is not None]
    mx = [c["sm_max_mhz"] for c in allc if c.get("sm_max_mhz") is not None]
    reasons = sorted({r for c in allc for r in c.get("reasons", [])})
    return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": min(mx) if mx else None,
            "reasons": reasons, "samples": sum(c.get("samples", 0) for c in allc), "per_rank": allc}


def env_rank():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1"))


# ---------------------------------------------------------------------------- oracle legs
def oracle_sample(cfg: StepConfig, n_spec: int = 8192, ccsdt_blocks: int = 1, threads: int | None = None):
    """Time the oracle (as it stands) on a bounded sample of the step: n_spec elements of
    each spectral kernel and `ccsdt_blocks` CCSD(T) blocks of d1+d2 fused.  Returns the
    step-equivalent GFLOP/s (each kernel's sample rate weighted by its share of the full
    step's flops), the sample description, the seconds spent and per-kernel GFLOP/s.
    Imports only oracle / synthetic / accounting."""
    import oracle
    import synthetic as syn

    if threads is not None:
        oracle.set_threads(threads)
    P1, t = cfg.P1, cfg.tile
    U = syn.elements(syn.TID["U"], P1, np.arange(n_spec))
    A, B, C = (syn.tensor(syn.TID[n], (P1, P1)) for n in ("A", "B", "C"))
    D = syn.gll_derivative(cfg.p)
    ext = (t,) * 7
    t3 = syn.tensor(syn.ccsdt_block_tid(syn.TID["T3"], 0, 0), (t ** 6,))
    ops = {fam: ([syn.tensor(syn.ccsdt_block_tid(syn.TID["T2"] + (0 if fam == "d1" else 200000), v, 0), (t ** 4,))
                  for v in range(1, 10)],
                 [syn.tensor(syn.ccsdt_block_tid(syn.TID["V2"] + (0 if fam == "d1" else 200000), v, 0), (t ** 4,))
                  for v in range(1, 10)]) for fam in cfg.families}
    secs = {}
    t0 = time.perf_counter(); oracle.local_grad3(D, U); secs["local_grad3"] = time.perf_counter() - t0
    t0 = time.perf_counter(); oracle.sumfact3d(A, B, C, U); secs["sumfact3d"] = time.perf_counter() - t0
    U2 = U.reshape(-1, P1, P1)
    t0 = time.perf_counter(); oracle.sumfact2d(A, B, U2); secs["sumfact2d"] = time.perf_counter() - t0
    for fam in cfg.families:
        t0 = time.perf_counter()
        for _ in range(ccsdt_blocks):
            oracle.ccsdt_fused(fam, ext, t3, *ops[fam])
        secs[f"ccsdt_{fam}_fused"] = time.perf_counter() - t0
    fb_s = acct.flops_bytes(cfg, n_spec)
    fb_f = acct.flops_bytes(cfg)
    sample_flops = {k: fb_s[k][0] * (ccsdt_blocks if k.startswith("ccsdt") else 1) for k in secs}
    full_flops = {k: fb_f[k][0] * (cfg.blocks if k.startswith("ccsdt") else 1) for k in secs}
    t_equiv = sum(secs[k] / sample_flops[k] * full_flops[k] for k in secs)
    rate = sum(full_flops.values()) / t_equiv / 1e9
    desc = (f"oracle (C, -O2, OpenMP) on {n_spec} of {cfg.n_elem} elements (p={cfg.p}) for local_grad3/"
            f"sumfact3d/sumfact2d and {ccsdt_blocks} of {cfg.blocks} tile-{t} blocks for CCSD(T) d1+d2 fused; "
            "each kernel's sample rate weighted by its flop share of the full step")
    return rate, desc, sum(secs.values()), {k: sample_flops[k] / secs[k] / 1e9 for k in secs}


def all_cores():
    n = os.environ.get("OMP_NUM_THREADS")
    return int(n) if n else len(os.sched_getaffinity(0))


def cpu_baseline(cfg, n_spec):
    """The oracle on all host cores and on one core (Table IV's "1 core" / "OpenMP"
    columns), with the CPU model."""
    cores = all_cores()
    rate, desc, secs, per = oracle_sample(cfg, n_spec=n_spec, threads=cores)
    rate1, _, secs1, per1 = oracle_sample(cfg, n_spec=max(256, n_spec // 8), threads=1)
    return {"value": rate, "unit": "GFLOP/s", "cores": cores, "kind": "oracle", "sample": desc,
            "cores_all": cores, "gflops_all": rate, "gflops_1core": rate1,
            "sample_1core": f"{max(256, n_spec // 8)} elements per spectral kernel, 1 block per CCSD(T) family",
            "cpu_model": cpu_model(), "seconds": secs + secs1, "per_kernel_gflops": per,
            "per_kernel_gflops_1core": per1}


def run_reference(args, cfg):
    """--impl reference: the oracle as it stands on the host cores (rank 0 only)."""
    rank, world = env_rank()
    if rank != 0:
        return
    cores = all_cores()
    for _ in range(args.warmup):
        oracle_sample(cfg, n_spec=args.ref_elems, threads=cores)
    rates, secs = [], 0.0
    desc = ""
    for _ in range(args.steps):
        r, desc, s, _ = oracle_sample(cfg, n_spec=args.ref_elems, threads=cores)
        rates.append(r)
        secs += s
    value = float(np.mean(rates))
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": secs / args.steps * 1e3,
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (counter-based splitmix64, seed 2015)",
        "config": workload_config(cfg, world, args.scaling),
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": cores, "kind": "oracle", "sample": desc,
                         "cpu_model": cpu_model()},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(cfg, world, scaling):
    per = "per GPU" if scaling == "weak" else f"global, sharded over {world} GPU(s)"
    return {
        "workload": f"BASELINE configs[1] Nekbone local_grad3 p={cfg.p} N={cfg.n_elem} ({per}) + the other hot-path "
                    f"rows on the same batch: sumfact3d (3-D, p={cfg.p}), sumfact2d (N*(p+1) 2-D elements), CCSD(T) "
                    f"{'+'.join(cfg.families)} 9-variant fused tile {cfg.tile} x {cfg.blocks} blocks ({per}), "
                    "check scalars",
        "p": cfg.p, "n_elem": cfg.n_elem, "ccsdt_tile": cfg.tile, "ccsdt_blocks": cfg.blocks,
        "scaling": scaling, "parallelism": f"elements+blocks sharded, dp{world}",
        "l2": "inputs larger than L2 (U alone is %.1f GB > 126 MB)" % (cfg.n_elem * cfg.P1 ** 3 * 8 / 1e9),
    }


# ---------------------------------------------------------------------------- GPU arm
def pipe_of(name: str, p: int) -> str:
    """FP64 pipe a kernel runs on (api.cu dispatch): the CCSD(T) TMA kernels and the
    spectral tensor-core kernels (P1 in {8, 15, 16}) issue DMMA, the rest DFMA."""
    if name.startswith("ccsdt"):
        return "dmma"
    return "dmma" if (p + 1) in (8, 15, 16) else "dfma"


def roof(fl, by, t_s, hbm_gbs, f64_tf, pipe):
    """Roofline fraction of one launch: t_bound / t_measured, bound = max(HBM, FP64)."""
    t_hbm, t_f64 = by / (hbm_gbs * 1e9), fl / (f64_tf[pipe] * 1e12)
    bound = "hbm" if t_hbm >= t_f64 else "alu"
    return {"gflops": fl / t_s / 1e9, "gbs": by / t_s / 1e9, "bound": bound, "pipe": pipe,
            "frac": (t_hbm if bound == "hbm" else t_f64) / t_s}


def time_calls(fn, inner: int, reps: int, stream) -> float:
    """Median ms per call of `inner` back-to-back calls, `reps` samples (after one warm call)."""
    fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(inner):
            fn()
        e1.record(stream)
        e1.synchronize()
        out.append(e0.elapsed_time(e1) / inner)
    return float(np.median(out))


def measure_configs(dev, hbm_gbs, f64_tf, stream):
    """BASELINE configs 1, 3, 4, 5 as rows: each kernel timed back to back
    with CUDA events on synthetic device-resident inputs; frac = roofline fraction."""
    import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
    import synthetic as syn
    f64 = torch.float64
    rows = {}

    # cfg 1: 3-D sumfact p=4, N=64 (latency-bound: 128.6 KB of traffic)
    P1, N = 5, 64
    ops = [bc.fill(torch.empty((P1, P1), dtype=f64, device=dev), syn.TID[n]) for n in ("A", "B", "C")]
    U = bc.fill(torch.empty((N, P1, P1, P1), dtype=f64, device=dev), syn.TID["U"])
    V = torch.empty_like(U)
    call = lambda: bc.sumfact3d(*ops, U, out=V)  # noqa: E731
    ms_call = time_calls(call, 200, 3, stream)
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream(dev)
    s.wait_stream(stream)
    with torch.cuda.stream(s):
        call()
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(100):
                call()
    stream.wait_stream(s)
    ms_graph = time_calls(g.replay, 5, 3, stream) / 100
    fl, by = acct.sumfact3d(P1, N)
    rows["cfg1_sumfact3d_p4_N64"] = {"us_per_call": ms_call * 1e3, "us_per_call_graph": ms_graph * 1e3,
                                     **roof(fl, by, ms_graph * 1e-3, hbm_gbs, f64_tf, pipe_of("sumfact3d", 4)),
                                     "note": "latency-bound: 16 ns of HBM time; frac shown for the graph-amortised call"}
    del U, V

    # cfg 3 / 4: CCSD(T) per variant and fused, tiles 16 and 24
    for fam, tiles in (("d1", (16, 24)), ("d2", (16, 24))):
        for t in tiles:
            ext = (t,) * 7
            t3 = bc.fill(torch.empty(t ** 6, dtype=f64, device=dev), 10)
            t2s = [bc.fill(torch.empty(t ** 4, dtype=f64, device=dev), 20 + v) for v in range(9)]
            v2s = [bc.fill(torch.empty(t ** 4, dtype=f64, device=dev), 40 + v) for v in range(9)]
            inner = 20 if t == 16 else 4
            per = []
            for v in range(1, 10):
                ms = time_calls(lambda: bc.ccsdt(fam, v, ext, t3, t2s[v - 1], v2s[v - 1]), inner, 3, stream)
                fl, by = acct.ccsdt_variants(ext, 1, fam)
                per.append({"variant": v, "us": ms * 1e3, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, "dmma")})
            fr = [r["frac"] for r in per]
            rows[f"cfg{3 if fam == 'd1' else 4}_{fam}_tile{t}_per_variant"] = {
                "us_min": min(r["us"] for r in per), "us_max": max(r["us"] for r in per),
                "frac_min": min(fr), "frac_median": float(np.median(fr)), "frac_max": max(fr),
                "bound": per[0]["bound"], "gflops_median": float(np.median([r["gflops"] for r in per]))}
            ms = time_calls(lambda: bc.ccsdt_fused(fam, ext, t3, t2s, v2s), max(2, inner // 4), 3, stream)
            fl, by = acct.ccsdt_variants(ext, 9, fam)
            rows[f"cfg{3 if fam == 'd1' else 4}_{fam}_tile{t}_fused9"] = {
                "us": ms * 1e3, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, "dmma")}
            del t3, t2s, v2s

    # NEXT rows: f1 local_grad3_t and f2 ax_e at p = 12, f3 s1 fused and
    # f4 (27 variants + energy, t3 never stored) at tiles 16 and 24
    p, P1 = 12, 13
    D = torch.from_numpy(syn.gll_derivative(p)).to(dev)
    N = 262144
    fields = [bc.fill(torch.empty((N, P1, P1, P1), dtype=f64, device=dev), 7 + i) for i in range(3)]
    W = torch.empty_like(fields[0])
    ms = time_calls(lambda: bc.local_grad3_t(D, *fields, out=W), 3, 3, stream)
    fl, by = acct.local_grad3_t(P1, N)
    rows[f"f1_local_grad3_t_p12_N{N}"] = {"ms": ms, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, pipe_of("lg3t", p))}
    del fields, W
    torch.cuda.empty_cache()
    N = 65536
    U = bc.fill(torch.empty((N, P1, P1, P1), dtype=f64, device=dev), syn.TID["U"])
    Gm = bc.fill(torch.empty((N, 6, P1, P1, P1), dtype=f64, device=dev), syn.TID["G"])
    W = torch.empty_like(U)
    ms = time_calls(lambda: bc.ax_e(D, U, Gm, out=W), 3, 3, stream)
    fl, by = acct.ax_e(P1, N)
    rows[f"f2_ax_e_p12_N{N}"] = {"ms": ms, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, pipe_of("ax_e", p))}
    del U, Gm, W
    torch.cuda.empty_cache()
    for t in (16, 24):
        ext = (t,) * 7
        t3 = bc.fill(torch.empty(t ** 6, dtype=f64, device=dev), 10)
        ops = {}
        for i, fam in enumerate(("s1", "d1", "d2")):
            na, nb = bc.operand_sizes(fam, ext)
            ops[fam] = ([bc.fill(torch.empty(na, dtype=f64, device=dev), 100 + 20 * i + v) for v in range(9)],
                        [bc.fill(torch.empty(nb, dtype=f64, device=dev), 110 + 20 * i + v) for v in range(9)])
        ms = time_calls(lambda: bc.ccsdt_fused("s1", ext, t3, *ops["s1"]), 8 if t == 16 else 2, 3, stream)
        fl, by = acct.ccsdt_variants(ext, 9, "s1")
        rows[f"f3_s1_tile{t}_fused9"] = {"us": ms * 1e3, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, "dfma")}
        eh = bc.fill(torch.empty(3 * t, dtype=f64, device=dev), syn.TID["EPS_H"], kind=bc.KIND_RANGE, lo=-2.0, hi=-0.5)
        ep = bc.fill(torch.empty(3 * t, dtype=f64, device=dev), syn.TID["EPS_P"], kind=bc.KIND_RANGE, lo=0.5, hi=2.0)
        ws = torch.empty(bc.BC_CHECK_WS_DOUBLES, dtype=f64, device=dev)
        ms = time_calls(lambda: bc.ccsdt_triples_energy(ext, ops["s1"], ops["d1"], ops["d2"], eh, ep, ws),
                        4 if t == 16 else 1, 3, stream)
        fl, by = acct.triples_energy(ext)
        rows[f"f4_triples_energy_tile{t}"] = {"us": ms * 1e3, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, "dmma")}
        del t3, ops
        torch.cuda.empty_cache()

    # cfg 5: spectral sweep at N = 2^22 (the largest point), 3-D and 2-D, p in {4, 8, 12}
    N = 1 << 22
    for p in (4, 8, 12):
        P1 = p + 1
        ops = [bc.fill(torch.empty((P1, P1), dtype=f64, device=dev), syn.TID[n]) for n in ("A", "B", "C")]
        for form in ("3d", "2d"):
            shape = (N, P1, P1, P1) if form == "3d" else (N, P1, P1)
            U = bc.fill(torch.empty(shape, dtype=f64, device=dev), syn.TID["U"])
            V = torch.empty_like(U)
            if form == "3d":
                fn = lambda: bc.sumfact3d(*ops, U, out=V)  # noqa: E731
                fl, by = acct.sumfact3d(P1, N)
                name = "sumfact3d"
            else:
                fn = lambda: bc.sumfact2d(ops[0], ops[1], U, out=V)  # noqa: E731
                fl, by = acct.sumfact2d(P1, N)
                name = "sumfact2d"
            ms = time_calls(fn, 3, 3, stream)
            rows[f"cfg5_{form}_p{p}_N{N}"] = {"ms": ms, **roof(fl, by, ms * 1e-3, hbm_gbs, f64_tf, pipe_of(name, p))}
            del U, V
            torch.cuda.empty_cache()
    return rows


def pcie_bandwidth(dev, stream, nbytes=1 << 30):
    """Pinned H2D / D2H copy bandwidth (GB/s) on this GPU: the e2e bound's denominators."""
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    out = {}
    for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))):
        ms = time_calls(fn, 2, 3, stream)
        out[name] = nbytes / (ms * 1e-3) / 1e9
    del h, d
    return out


def measure_e2e(args, step, rank, dev, stream, flops_all, ref_checks):
    """The same step through the public API with every input copied in from pinned host
    memory and every output (ur, us, ut, V, V2, all t3 blocks, the check scalars) copied
    back, each step, overlapped by HostPipeline (timed on the device, max over ranks)."""
    from paper_conf_icpp_nelsonrbhhjn15_b200 import dist as bdist
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import HostPipeline
    t0 = time.perf_counter()
    pipe = HostPipeline(step, chunks=args.e2e_chunks)
    pin_s = time.perf_counter() - t0
    bw = pcie_bandwidth(dev, stream)
    pipe.run()
    torch.cuda.synchronize(dev)
    bdist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    pipe.fork(stream)
    for _ in range(args.e2e_steps):
        pipe.run()
    pipe.join(stream)
    e1.record(stream)
    torch.cuda.synchronize(dev)
    ms = bdist.max_over_ranks(e0.elapsed_time(e1) / args.e2e_steps, dev)
    # results that reached the host: sum V^2 vs the device-resident step's (same inputs and
    # kernels; reduced per chunk here, so equal to rounding), and the last chunk / t3 block
    # in the host ring bitwise equal to the device copies
    rel = abs(pipe.h_chk[0].item() - ref_checks[0].item()) / abs(ref_checks[0].item())
    a, b = pipe.bounds[-1]
    ci = len(pipe.bounds) - 1
    host_ok = all(torch.equal(pipe.h_ring[nm][ci % pipe.out_slots][:b - a], getattr(step, nm)[a:b].cpu())
                  for nm in ("ur", "us", "ut", "V"))
    if step.nb:
        host_ok = host_ok and torch.equal(pipe.h_t3[(step.nb - 1) % len(pipe.h_t3)], step.t3[-1].cpu())
    t_bound = max(pipe.h2d_bytes / (bw["h2d"] * 1e9), pipe.d2h_bytes / (bw["d2h"] * 1e9))
    out = {"value": flops_all / (ms * 1e-3) / 1e9, "unit": "GFLOP/s",
           "h2d_bytes_per_step": int(pipe.h2d_bytes), "d2h_bytes_per_step": int(pipe.d2h_bytes),
           "ms_per_step": ms, "pcie_gbs": bw, "pcie_bound_ms": t_bound * 1e3,
           "frac_of_pcie_bound": t_bound * 1e3 / ms, "pinned_setup_s": pin_s,
           "sumsq_rel_diff_vs_device_step": rel, "host_results_match_device": bool(host_ok),
           "host_outputs": f"ring of {pipe.out_slots} pinned chunk slots per output", "chunks": args.e2e_chunks,
           "api": "paper_conf_icpp_nelsonrbhhjn15_b200 (ctypes -> libbarracuda C ABI), pinned host inputs and "
                  "outputs, H2D / compute / D2H on three streams"}
    del pipe
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="barracuda", choices=["barracuda", "reference"])
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    ap.add_argument("--p", type=int, default=12)
    ap.add_argument("--n-elem", type=int, default=262144)
    ap.add_argument("--tile", type=int, default=16)
    ap.add_argument("--blocks", type=int, default=8)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--e2e-chunks", type=int, default=16)
    ap.add_argument("--ref-elems", type=int, default=8192)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-configs", action="store_true")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    cfg = StepConfig(p=args.p, n_elem=args.n_elem, tile=args.tile, blocks=args.blocks)

    if args.impl == "reference":
        run_reference(args, cfg)
        return

    from paper_conf_icpp_nelsonrbhhjn15_b200 import dist as bdist
    rank = bdist.init()
    import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import Step

    dev = rank.device
    stream = torch.cuda.current_stream(dev)
    # FP64 roofline denominators, measured live on this GPU
    f64_tf, f64_src = {}, "live probe (bc_probe_fp64): best of 3 launches, 8 CTAs x 512 threads per SM"
    try:
        f64_tf = {k: bc.probe_fp64_tflops(k, dev) for k in ("dfma", "dmma")}
    except Exception as exc:  # noqa: BLE001
        f64_tf = {"dfma": FP64_NOMINAL_TFLOPS, "dmma": FP64_NOMINAL_TFLOPS}
        f64_src = f"nominal 148x64x2x1.965 GHz (probe failed: {exc})"

    step = Step(cfg, rank.rank, rank.world, dev, scaling=args.scaling)
    torch.cuda.synchronize(dev)
    for _ in range(args.warmup):
        step.run()
    torch.cuda.synchronize(dev)

    # ---- device-resident timed region: K steps, per-kernel events on the launching stream
    names = list(step.launches_per_step().keys())
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(len(names) + 1)] for _ in range(args.steps)]
    bdist.barrier()
    torch.cuda.synchronize(dev)
    bc.reset_launch_count()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev.index or 0) as clocks:
        start.record(stream)
        for s in range(args.steps):
            ev[s][0].record(stream)
            idx = [0]

            def tick(name, s=s):
                idx[0] += 1
                ev[s][idx[0]].record(stream)
            step.run(timer=tick)
        end.record(stream)
        torch.cuda.synchronize(dev)
    launches = bc.launch_count()
    bdist.barrier()
    ms_local = start.elapsed_time(end) / args.steps
    ms = bdist.max_over_ranks(ms_local, dev)
    per_kernel_ms = {n: float(np.mean([ev[s][i].elapsed_time(ev[s][i + 1]) for s in range(args.steps)]))
                     for i, n in enumerate(names)}

    flops_local = step.flops_per_step()
    flops_all = bdist.sum_over_ranks(flops_local, dev)
    value = flops_all / (ms * 1e-3) / 1e9

    # ---- roofline of the dominant kernel (largest share of the step)
    hbm_gbs, hbm_src = load_peaks()
    lps = step.launches_per_step()
    kernels = {}
    for n in names:
        if n.startswith("check") or not lps[n]:
            continue
        fl, by = step.fb[n]
        t_launch = per_kernel_ms[n] / lps[n] * 1e-3
        kernels[n] = {"ms_per_step": per_kernel_ms[n], "launches": lps[n],
                      **roof(fl, by, t_launch, hbm_gbs, f64_tf, pipe_of(n, cfg.p))}
    dom = max(kernels, key=lambda n: kernels[n]["ms_per_step"])
    k = kernels[dom]
    traffic = load_traffic().get(f"{dom}:p{cfg.p}:n{step.n}:t{cfg.tile}")
    if k["bound"] == "hbm":
        roofline = {"kernel": dom, "bound": "hbm", "achieved": k["gbs"], "peak": hbm_gbs, "unit": "GB/s",
                    "frac": k["frac"], "traffic": traffic, "peak_source": hbm_src,
                    "algorithmic_bytes_per_launch": step.fb[dom][1]}
    else:
        roofline = {"kernel": dom, "bound": "alu", "achieved": k["gflops"] / 1e3, "peak": f64_tf[k["pipe"]],
                    "unit": "TFLOP/s", "frac": k["frac"], "traffic": traffic,
                    "peak_source": f"{k['pipe'].upper()} {f64_src}",
                    "algorithmic_flops_per_launch": step.fb[dom][0]}

    # ---- end to end: pinned host inputs in, every output out, each step (overlapped)
    e2e = None
    if not args.no_e2e:
        try:
            e2e = measure_e2e(args, step, rank, dev, stream, flops_all, step.checks.cpu().clone())
        except (RuntimeError, MemoryError) as exc:  # e.g. pinned host memory exhausted with many ranks
            e2e = {"value": None, "unit": "GFLOP/s", "error": f"{type(exc).__name__}: {str(exc)[:160]}"}
    clk = gather_clocks(clocks.summary(), rank)
    del step
    torch.cuda.empty_cache()

    configs = None
    if rank.rank == 0 and rank.world == 1 and not args.no_configs:
        configs = measure_configs(dev, hbm_gbs, f64_tf, stream)

    cpu = None
    if rank.rank == 0 and rank.world == 1 and not args.no_cpu:
        cpu = cpu_baseline(cfg, args.ref_elems)

    if rank.rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": rank.world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": args.scaling,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic (counter-based splitmix64, seed 2015)",
            "config": workload_config(cfg, rank.world, args.scaling),
            "roofline": roofline, "kernels": kernels, "gpu_launches": int(launches),
            "fp64_peak_tflops": {**f64_tf, "source": f64_src},
            "clocks": clk, "e2e": e2e, "configs": configs, "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    bdist.finalize()


if __name__ == "__main__":
    main()
