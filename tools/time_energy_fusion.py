"""A/B on one box: CCSD(T) part of the bench step (8 tile-16 blocks, d1 then d2 fused) with
the energy check as a separate pass vs fused into d2 (bc_ccsdt_fused_energy)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t, nb = 16, 8
ext = (t,) * 7
f64, dev = torch.float64, "cuda"
t3 = [bc.fill(torch.empty(t ** 6, dtype=f64, device=dev), 10 + 100 * b) for b in range(nb)]
ops = {f: ([bc.fill(torch.empty(t ** 4, dtype=f64, device=dev), 20 + v + k) for v in range(9)],
           [bc.fill(torch.empty(t ** 4, dtype=f64, device=dev), 40 + v + k) for v in range(9)])
       for f, k in (("d1", 0), ("d2", 200000))}
eh = bc.fill(torch.empty(3 * t, dtype=f64, device=dev), 60, kind=bc.KIND_RANGE, lo=-2.0, hi=-0.5)
ep = bc.fill(torch.empty(3 * t, dtype=f64, device=dev), 61, kind=bc.KIND_RANGE, lo=0.5, hi=2.0)
ws = torch.empty((nb, bc.BC_CHECK_WS_DOUBLES), dtype=f64, device=dev)


def separate():
    for b in range(nb):
        bc.ccsdt_fused("d1", ext, t3[b], *ops["d1"])
    for b in range(nb):
        bc.ccsdt_fused("d2", ext, t3[b], *ops["d2"])
    for b in range(nb):
        bc.check_energy(ext, t3[b], eh, ep, ws[b])


def fused():
    for b in range(nb):
        bc.ccsdt_fused("d1", ext, t3[b], *ops["d1"])
    for b in range(nb):
        bc.ccsdt_fused_energy("d2", ext, t3[b], *ops["d2"], eh, ep, ws[b])


def timeit(fn, reps=10):
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); [fn() for _ in range(reps)]; e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


res = {"separate_ms": [], "fused_ms": []}
for _ in range(3):
    res["separate_ms"].append(round(timeit(separate), 4))
    res["fused_ms"].append(round(timeit(fused), 4))
print(json.dumps(res))
