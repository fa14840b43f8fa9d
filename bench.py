#!/usr/bin/env python3
"""Benchmark: fp64 GFLOP/s of one pass of the whole hot path.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl barracuda|reference]

N > 1 is launched by the driver with torchrun (one process per GPU, NCCL).  Each rank owns
its own slice of the global batch (weak scaling; no data-path collective — only the
check-scalar SUM and the max-over-ranks of the timing cross GPUs).  Rank 0 prints ONE JSON
line.  The default workload is BASELINE.json configs[1] (Nekbone local_grad3, p=12,
N=262,144 elements per GPU) with every other §8(a) row run over the same batch in the same
step (sumfact3d, sumfact2d, CCSD(T) d1/d2 fused tile 16, check scalars).

Only the cpu_baseline leg and --impl reference execute the oracle (oracle/), on host cores.
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

FP64_PEAK_TFLOPS = 37.2  # 148 SMs x 64 FP64 FMA/clk x 2 x 1.965 GHz; measured 37.1 (DMMA) / 34.2 (DFMA),
#                          tools/fp64_peak.cu -> profiles/fp64_peak_r01.txt
METRIC = "fp64 GFLOP/s & % of HBM/FP64 roofline for batched small contractions, 1-8 GPU"


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
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(mx), "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------- oracle legs
def oracle_sample_rate(cfg, n_spec: int = 8192, ccsdt_blocks: int = 1):
    """Time the oracle (as it stands) on a bounded sample of the step and return the
    step-equivalent GFLOP/s (each kernel's sample rate weighted by its share of the full
    step's flops), the sample description and the seconds spent."""
    import oracle
    import synthetic as syn
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import flops_bytes

    P1 = cfg.P1
    fb = flops_bytes(cfg)
    U = syn.elements(syn.TID["U"], P1, np.arange(n_spec))
    A, B, C = (syn.tensor(syn.TID[n], (P1, P1)) for n in ("A", "B", "C"))
    D = syn.gll_derivative(cfg.p)
    t = cfg.tile
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
    sample_flops = {"local_grad3": fb["local_grad3"][0] * n_spec / cfg.n_elem,
                    "sumfact3d": fb["sumfact3d"][0] * n_spec / cfg.n_elem,
                    "sumfact2d": fb["sumfact2d"][0] * n_spec / cfg.n_elem,
                    **{f"ccsdt_{f}_fused": fb[f"ccsdt_{f}_fused"][0] * ccsdt_blocks for f in cfg.families}}
    full_flops = {k: fb[k][0] * (cfg.blocks if k.startswith("ccsdt") else 1) for k in sample_flops}
    t_equiv = sum(secs[k] / sample_flops[k] * full_flops[k] for k in secs)
    rate = sum(full_flops.values()) / t_equiv / 1e9
    desc = (f"oracle (C, -O2, OpenMP) on {n_spec} of {cfg.n_elem} elements (p={cfg.p}) for local_grad3/"
            f"sumfact3d/sumfact2d and {ccsdt_blocks} of {cfg.blocks} tile-{t} blocks for CCSD(T) d1+d2 fused; "
            "each kernel's sample rate weighted by its flop share of the full step")
    return rate, desc, sum(secs.values()), {k: sample_flops[k] / secs[k] / 1e9 for k in secs}


def threads_used():
    n = os.environ.get("OMP_NUM_THREADS")
    return int(n) if n else len(os.sched_getaffinity(0))


def run_reference(args, cfg, rank):
    """--impl reference: the oracle as it stands on the host cores (rank 0 only)."""
    if rank.rank != 0:
        return
    for _ in range(args.warmup):
        oracle_sample_rate(cfg, n_spec=args.ref_elems)
    rates, secs = [], 0.0
    for _ in range(args.steps):
        r, desc, s, _ = oracle_sample_rate(cfg, n_spec=args.ref_elems)
        rates.append(r)
        secs += s
    value = float(np.mean(rates))
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": rank.world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": secs / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(cfg, rank.world),
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": threads_used(), "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(cfg, world):
    return {
        "workload": f"BASELINE configs[1] Nekbone local_grad3 p={cfg.p} N={cfg.n_elem}/GPU + the other hot-path rows "
                    f"on the same batch: sumfact3d (3-D, p={cfg.p}), sumfact2d (N*(p+1) 2-D elements), CCSD(T) "
                    f"{'+'.join(cfg.families)} 9-variant fused tile {cfg.tile} x {cfg.blocks} blocks/GPU, check scalars",
        "p": cfg.p, "n_elem_per_gpu": cfg.n_elem, "ccsdt_tile": cfg.tile, "ccsdt_blocks_per_gpu": cfg.blocks,
        "parallelism": f"elements+blocks sharded, dp{world}",
        "l2": "inputs larger than L2 (U alone is %.1f GB > 126 MB)" % (cfg.n_elem * cfg.P1 ** 3 * 8 / 1e9),
    }


def measure_e2e(args, step, rank, dev, stream, flops_step):
    """Same step through the public API with every input copied from pinned host memory
    each step and the check scalars read back (timed on the device, max over ranks)."""
    from paper_conf_icpp_nelsonrbhhjn15_b200 import dist as bdist
    ins = step.inputs()
    host = [torch.empty(t.shape, dtype=t.dtype, pin_memory=True) for t in ins]
    for h, t in zip(host, ins):
        h.copy_(t)
    out_host = torch.empty(2, dtype=torch.float64, pin_memory=True)
    h2d = sum(t.numel() * t.element_size() for t in ins)
    torch.cuda.synchronize(dev)

    def e2e_step():
        for h, t in zip(host, ins):
            t.copy_(h, non_blocking=True)
        chk = step.run()
        out_host.copy_(chk, non_blocking=True)

    e2e_step()
    torch.cuda.synchronize(dev)
    bdist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.e2e_steps):
        e2e_step()
    e1.record(stream)
    torch.cuda.synchronize(dev)
    ems = bdist.max_over_ranks(e0.elapsed_time(e1) / args.e2e_steps, dev)
    return {"value": flops_step * rank.world / (ems * 1e-3) / 1e9, "unit": "GFLOP/s",
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": 16, "ms_per_step": ems,
            "api": "paper_conf_icpp_nelsonrbhhjn15_b200 (ctypes -> libbarracuda C ABI), pinned host inputs"}


# ---------------------------------------------------------------------------- main arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="barracuda", choices=["barracuda", "reference"])
    ap.add_argument("--p", type=int, default=12)
    ap.add_argument("--n-elem", type=int, default=262144)
    ap.add_argument("--tile", type=int, default=16)
    ap.add_argument("--blocks", type=int, default=8)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--ref-elems", type=int, default=8192)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    from paper_conf_icpp_nelsonrbhhjn15_b200 import dist as bdist
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import StepConfig

    cfg = StepConfig(p=args.p, n_elem=args.n_elem, tile=args.tile, blocks=args.blocks)
    if args.impl == "reference":
        world = int(os.environ.get("WORLD_SIZE", "1"))
        rank = bdist.Rank(int(os.environ.get("RANK", "0")), world, int(os.environ.get("LOCAL_RANK", "0")),
                          torch.device("cpu"))
        run_reference(args, cfg, rank)
        return

    rank = bdist.init()
    import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import Step

    dev = rank.device
    step = Step(cfg, rank.rank, rank.world, dev)
    stream = torch.cuda.current_stream(dev)
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

    flops_step = step.flops_per_step()
    value = flops_step * rank.world / (ms * 1e-3) / 1e9

    # ---- roofline of the dominant kernel (largest share of the step)
    hbm_gbs, hbm_src = load_peaks()
    lps = step.launches_per_step()
    kernels = {}
    for n in names:
        if n.startswith("check"):
            continue
        fl, by = step.fb[n]
        t_launch = per_kernel_ms[n] / lps[n] * 1e-3
        t_hbm, t_f64 = by / (hbm_gbs * 1e9), fl / (FP64_PEAK_TFLOPS * 1e12)
        bound = "hbm" if t_hbm >= t_f64 else "alu"
        kernels[n] = {"ms_per_step": per_kernel_ms[n], "launches": lps[n], "gflops": fl / t_launch / 1e9,
                      "gbs": by / t_launch / 1e9, "bound": bound,
                      "frac": (by / t_launch / 1e9 / hbm_gbs) if bound == "hbm" else (fl / t_launch / 1e12 / FP64_PEAK_TFLOPS)}
    dom = max(kernels, key=lambda n: kernels[n]["ms_per_step"])
    k = kernels[dom]
    traffic = load_traffic().get(f"{dom}:p{cfg.p}:n{cfg.n_elem}:t{cfg.tile}")
    if k["bound"] == "hbm":
        roof = {"kernel": dom, "bound": "hbm", "achieved": k["gbs"], "peak": hbm_gbs, "unit": "GB/s",
                "frac": k["frac"], "traffic": traffic, "peak_source": hbm_src,
                "algorithmic_bytes_per_launch": step.fb[dom][1]}
    else:
        roof = {"kernel": dom, "bound": "alu", "achieved": k["gflops"] / 1e3, "peak": FP64_PEAK_TFLOPS,
                "unit": "TFLOP/s", "frac": k["frac"], "traffic": traffic,
                "peak_source": "FP64 148x64x2x1.965GHz (measured DMMA 37.1 / DFMA 34.2, profiles/fp64_peak_r01.txt)",
                "algorithmic_flops_per_launch": step.fb[dom][0]}

    # ---- end to end: host (pinned) inputs copied in every step, check scalars copied out
    e2e = None
    if not args.no_e2e:
        try:
            e2e = measure_e2e(args, step, rank, dev, stream, flops_step)
        except (RuntimeError, MemoryError) as exc:  # e.g. pinned host memory exhausted with many ranks
            e2e = {"value": None, "unit": "GFLOP/s", "error": f"{type(exc).__name__}: {str(exc)[:160]}"}

    cpu = None
    if rank.rank == 0 and rank.world == 1 and not args.no_cpu:
        rate, desc, secs, per = oracle_sample_rate(cfg, n_spec=args.ref_elems)
        cpu = {"value": rate, "unit": "GFLOP/s", "cores": threads_used(), "kind": "oracle", "sample": desc,
               "seconds": secs, "per_kernel_gflops": per}

    if rank.rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": rank.world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic (counter-based splitmix64, seed 2015)",
            "config": workload_config(cfg, rank.world),
            "roofline": roof, "kernels": kernels, "gpu_launches": int(launches),
            "clocks": clocks.summary(), "e2e": e2e, "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    bdist.finalize()


if __name__ == "__main__":
    main()
