"""Per-row / per-config measurements (BASELINE.json configs 1-5 and the NEXT rows), one
JSON line each: time (CUDA events, median of R calls after warm-up, inputs > L2 or a
flush between calls), GFLOP/s, units/s, and the roofline fraction of the kernel's bound.

    python tools/bench_rows.py [--quick] > profiles/rows_rNN.jsonl

Roofline: HBM = MEASURED_PEAKS.json hbm_gbs; FP64 = 37.2 TFLOP/s (bench.py).  Bound =
max(bytes/HBM, flops/FP64) with the algorithmic bytes/flops of DESIGN.md §4.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_icpp_nelsonrbhhjn15_b200 as bc  # noqa: E402
import synthetic as syn  # noqa: E402

HBM = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
F64 = 37.2
DEV = torch.device("cuda")
FLUSH = torch.empty(256 * 1024 * 1024 // 8, dtype=torch.float64, device=DEV)  # 256 MiB > L2


def timed(fn, reps=20, flush=False, inner=None):
    """Median / mean ms per call.  `inner` calls are queued back to back between the two
    events, so the host-side cost of a call (Python, ctypes, validation, launch) overlaps
    the previous call's kernel instead of being timed as GPU idle time (default: enough
    calls for ~2 ms per sample)."""
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    if inner is None:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(5):
            fn()
        e1.record()
        torch.cuda.synchronize()
        inner = max(1, min(200, int(2.0 / max(e0.elapsed_time(e1) / 5, 1e-3))))
    ts = []
    for _ in range(reps):
        if flush:
            FLUSH.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(inner):
            fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / inner)
    return statistics.median(ts), statistics.mean(ts)


def emit(name, cfg, ms, mean_ms, flops, nbytes, units, unit_name, extra=None):
    t_hbm, t_f64 = nbytes / (HBM * 1e9), flops / (F64 * 1e12)
    bound = "hbm" if t_hbm >= t_f64 else "fp64"
    frac = max(t_hbm, t_f64) / (ms * 1e-3)
    d = {"row": name, "config": cfg, "ms": round(ms, 5), "mean_ms": round(mean_ms, 5),
         "gflops": round(flops / ms / 1e6, 1), "gbs": round(nbytes / ms / 1e6, 1),
         unit_name: round(units / (ms * 1e-3), 1), "bound": bound, "roofline_frac": round(frac, 3)}
    if extra:
        d.update(extra)
    print(json.dumps(d), flush=True)


def spectral(p, N, dims):
    P1 = p + 1
    shape = (N,) + (P1,) * dims
    U = bc.fill(torch.empty(shape, dtype=torch.float64, device=DEV), 1)
    A, B, C = (bc.fill(torch.empty((P1, P1), dtype=torch.float64, device=DEV), t) for t in (2, 3, 4))
    return P1, U, A, B, C


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--sections", default="cfg1,cfg5,cfg2,ccsdt", help="comma list of cfg1,cfg5,cfg2,ccsdt")
    ap.add_argument("--tiles", default="16,24")
    args = ap.parse_args()
    sec = set(args.sections.split(","))
    if "cfg1" in sec:
        cfg1()
    if "cfg5" in sec:
        cfg5(args)
    if "cfg2" in sec:
        cfg2()
    if "ccsdt" in sec:
        ccsdt(args)


def cfg1():

    # ---- config 1: 3-D p=4, N=64 (latency-bound by construction): per call and graph-amortised
    P1, U, A, B, C = spectral(4, 64, 3)
    V = torch.empty_like(U)
    ms, mean = timed(lambda: bc.sumfact3d(A, B, C, U, out=V), reps=200, inner=1)
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        bc.sumfact3d(A, B, C, U, out=V)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(1000):
                bc.sumfact3d(A, B, C, U, out=V)
    torch.cuda.synchronize()
    gms, _ = timed(lambda: g.replay(), reps=5, inner=1)
    emit("sumfact3d", "cfg1 p=4 N=64", ms, mean, 6 * P1 ** 4 * 64, 16 * P1 ** 3 * 64, 64, "elements_per_s",
         {"graph_us_per_call": round(gms * 1e3 / 1000, 3), "note": "HBM time 16 ns: launch/latency-bound"})



def cfg5(args):
    # ---- config 5: spectral sweep p = 4..12, N = 2^16 .. 2^22, 3-D and 2-D
    ps = [4, 8, 12] if args.quick else [4, 5, 6, 7, 8, 9, 10, 11, 12]
    Ns = [2 ** 20] if args.quick else [2 ** 16, 2 ** 18, 2 ** 20, 2 ** 22]
    free = torch.cuda.mem_get_info()[0]
    for p in ps:
        for N in Ns:
            P1 = p + 1
            if 2.2 * N * P1 ** 3 * 8 < free:
                P1, U, A, B, C = spectral(p, N, 3)
                V = torch.empty_like(U)
                ms, mean = timed(lambda: bc.sumfact3d(A, B, C, U, out=V), reps=10, flush=N * P1 ** 3 * 8 < 2e8)
                emit("sumfact3d", f"cfg5 3-D p={p} N={N}", ms, mean, 6 * P1 ** 4 * N, 16 * P1 ** 3 * N, N,
                     "elements_per_s")
                del U, V
                torch.cuda.empty_cache()
            P1, U, A, B, C = spectral(p, N, 2)
            V = torch.empty_like(U)
            ms, mean = timed(lambda: bc.sumfact2d(A, B, U, out=V), reps=10, flush=N * P1 ** 2 * 8 < 2e8)
            emit("sumfact2d", f"cfg5 2-D p={p} N={N}", ms, mean, 4 * P1 ** 3 * N, 16 * P1 ** 2 * N, N, "elements_per_s")
            del U, V
            torch.cuda.empty_cache()



def cfg2():
    # ---- config 2: local_grad3 p=12 N=262144, and the NEXT rows at the same size
    p, N = 12, 262144
    P1, U, A, B, C = spectral(p, N, 3)
    D = torch.from_numpy(syn.gll_derivative(p)).to(DEV)
    outs = tuple(torch.empty_like(U) for _ in range(3))
    ms, mean = timed(lambda: bc.local_grad3(D, U, out=outs), reps=10)
    emit("local_grad3", "cfg2 p=12 N=262144", ms, mean, 6 * P1 ** 4 * N, 32 * P1 ** 3 * N, N, "elements_per_s")
    W = torch.empty_like(U)
    ms, mean = timed(lambda: bc.local_grad3_t(D, *outs, out=W), reps=10)
    emit("local_grad3_t", "f1 p=12 N=262144", ms, mean, 6 * P1 ** 4 * N + 2 * P1 ** 3 * N, 32 * P1 ** 3 * N, N,
         "elements_per_s")
    del outs
    torch.cuda.empty_cache()
    Ng = N // 4
    Gm = bc.fill(torch.empty((Ng, 6, P1, P1, P1), dtype=torch.float64, device=DEV), 11)
    Ug, Wg = U[:Ng], W[:Ng]
    ms, mean = timed(lambda: bc.ax_e(D, Ug, Gm, out=Wg), reps=10)
    emit("ax_e", f"f2 p=12 N={Ng}", ms, mean, (12 * P1 ** 4 + 17 * P1 ** 3) * Ng, 64 * P1 ** 3 * Ng, Ng,
         "elements_per_s")
    del U, W, Gm, Ug, Wg
    torch.cuda.empty_cache()



def ccsdt(args):
    # ---- configs 3 / 4: CCSD(T) per-variant and fused, tiles 16 and 24 (s1: NEXT f3)
    for t in ([16] if args.quick else [int(x) for x in args.tiles.split(",")]):
        ext = (t,) * 7
        t3 = bc.fill(torch.empty(t ** 6, dtype=torch.float64, device=DEV), 10)
        ops = {f: ([bc.fill(torch.empty(t ** 4, dtype=torch.float64, device=DEV), 20 + v) for v in range(9)],
                   [bc.fill(torch.empty(t ** 4, dtype=torch.float64, device=DEV), 40 + v) for v in range(9)])
               for f in ("d1", "d2")}
        n3 = t ** 6
        for f in ("d1", "d2"):
            for v in (1, 5, 9) if args.quick else range(1, 10):
                ms, mean = timed(lambda: bc.ccsdt(f, v, ext, t3, ops[f][0][v - 1], ops[f][1][v - 1]), reps=10)
                emit(f"ccsdt_{f}", f"cfg{3 if f == 'd1' else 4} tile={t} variant={v}", ms, mean, 2.0 * n3 * t,
                     16.0 * n3 + 16.0 * t ** 4, 1, "tiles_per_s")
            ms, mean = timed(lambda: bc.ccsdt_fused(f, ext, t3, *ops[f]), reps=10)
            emit(f"ccsdt_{f}_fused", f"cfg{3 if f == 'd1' else 4} tile={t} 9 variants fused", ms, mean,
                 18.0 * n3 * t, 16.0 * n3 + 9 * 16.0 * t ** 4, 1, "tiles_per_s")
        t1s = [bc.fill(torch.empty(t * t, dtype=torch.float64, device=DEV), 50 + v) for v in range(9)]
        ms, mean = timed(lambda: bc.ccsdt_fused("s1", ext, t3, t1s, ops["d1"][1]), reps=10)
        emit("ccsdt_s1_fused", f"f3 tile={t} 9 variants fused", ms, mean, 9 * 2.0 * n3, 16.0 * n3 + 9 * 8.0 * (t * t + t ** 4),
             1, "tiles_per_s")
        eh = bc.fill(torch.empty(3 * t, dtype=torch.float64, device=DEV), 60, kind=bc.KIND_RANGE, lo=-2.0, hi=-0.5)
        ep = bc.fill(torch.empty(3 * t, dtype=torch.float64, device=DEV), 61, kind=bc.KIND_RANGE, lo=0.5, hi=2.0)
        ws = torch.empty(1024, dtype=torch.float64, device=DEV)
        ms, mean = timed(lambda: bc.ccsdt_triples_energy(ext, (t1s, ops["d1"][1]), ops["d1"], ops["d2"], eh, ep, ws),
                         reps=10)
        emit("ccsdt_triples_energy", f"f4 tile={t} 27 variants + energy, t3 never stored", ms, mean,
             (36.0 * t + 18.0 + 4.0) * n3, 9 * 8.0 * (t * t + t ** 4) + 18 * 16.0 * t ** 4, 1, "tiles_per_s")
        del t3, ops, t1s
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
