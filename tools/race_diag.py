"""Repeat-run race diagnostic for the fused tile-16 CCSD(T) TMA kernel (GPU; builder tool).

Runs the determinism test's configuration (tile 16, B blocks, all 9 variants of d1 then
d2) R times on identical inputs with the library in $BARRACUDA_LIB, takes the elementwise
majority of the first three runs as the reference, and for every run that differs writes
the differing positions decoded into (block, particle plane, q0, q1, q2) with the good and
bad values.  One JSON line per library on stdout; details to --dump.

usage: BARRACUDA_LIB=... python tools/race_diag.py --repeats 60 --dump gpurun_out/x.json
"""
import argparse
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--repeats", type=int, default=40)
    ap.add_argument("--blocks", type=int, default=8)
    ap.add_argument("--tile", type=int, default=16)
    ap.add_argument("--fams", default="d1,d2")
    ap.add_argument("--dump", default=None)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    f64 = torch.float64
    t = a.tile
    ext = (t,) * 7
    fams = a.fams.split(",")
    base = [bc.fill(torch.empty(t ** 6, dtype=f64, device=dev), 10 + 100 * b) for b in range(a.blocks)]
    ops = {f: ([bc.fill(torch.empty(t ** 4, dtype=f64, device=dev), 20 + v + 50 * i) for v in range(9)],
               [bc.fill(torch.empty(t ** 4, dtype=f64, device=dev), 40 + v + 50 * i) for v in range(9)])
           for i, f in enumerate(("d1", "d2"))}
    ref_d = None
    first = []
    bad_runs, details = [], []
    t0 = time.time()
    times = []

    def compare(r, xd):
        diff = (xd != ref_d)
        n = int(diff.sum().item())
        if not n:
            return
        bad_runs.append({"run": r, "ndiff": n})
        if len(details) > 2048:
            return
        idx = diff.nonzero()
        for bi, fi in idx[:256].tolist():
            q, rem = [], fi
            for _ in range(6):
                q.append(rem % t)
                rem //= t
            details.append({"run": r, "block": bi, "flat": fi, "q": q, "good": float(ref_d[bi, fi]),
                            "bad": float(xd[bi, fi])})

    for r in range(a.repeats):
        t3 = [x.clone() for x in base]
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record()
        for f in fams:
            for b in range(a.blocks):
                bc.ccsdt_fused(f, ext, t3[b], *ops[f])
        ev1.record()
        torch.cuda.synchronize()
        times.append(ev0.elapsed_time(ev1))
        x = torch.stack(t3)
        del t3
        if r < 3:
            first.append(x)
            if r == 2:  # reference: elementwise majority of runs 0..2
                ref_d = torch.where(first[0] == first[1], first[0], first[2])
                for rr, xx in enumerate(first):
                    compare(rr, xx)
                first = []
            continue
        compare(r, x)
    out = {"lib": os.path.basename(bc.LIB_PATH), "repeats": a.repeats, "fams": fams, "blocks": a.blocks,
           "bad_runs": bad_runs, "n_bad_runs": len(bad_runs), "ms_median": sorted(times)[len(times) // 2],
           "wall_s": round(time.time() - t0, 1)}
    print(json.dumps(out), flush=True)
    if a.dump:
        with open(a.dump, "w") as fh:
            json.dump({"summary": out, "details": details}, fh)


if __name__ == "__main__":
    main()
