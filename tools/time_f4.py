"""Time the f4 kernel (27 variants + energy, one full tile block: extents TILE^7) for a
given build (BARRACUDA_LIB); prints one JSON line (ms per block, fraction of the nominal
FP64 peak over the d1 + d2 flops)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t = int(os.environ.get("TILE", "16"))
ext = (t,) * 7
dev = "cuda"
def ops(base, n):
    return [bc.fill(torch.empty(n, dtype=torch.float64, device=dev), base + v) for v in range(9)]
s1 = (ops(50, t * t), ops(70, t ** 4))
d1 = (ops(20, t ** 4), ops(40, t ** 4))
d2 = (ops(200020, t ** 4), ops(200040, t ** 4))
eh = bc.fill(torch.empty(3 * t, dtype=torch.float64, device=dev), 60, kind=bc.KIND_RANGE, lo=-2.0, hi=-0.5)
ep = bc.fill(torch.empty(3 * t, dtype=torch.float64, device=dev), 61, kind=bc.KIND_RANGE, lo=0.5, hi=2.0)
ws = torch.empty(bc.BC_CHECK_WS_DOUBLES, dtype=torch.float64, device=dev)
run = lambda: bc.ccsdt_triples_energy(ext, s1, d1, d2, eh, ep, ws=ws)  # noqa: E731
run(); torch.cuda.synchronize()
reps = 20 if t == 16 else 3
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); [run() for _ in range(reps)]; e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
fl = 36.0 * t ** 7
print(json.dumps({"lib": os.path.basename(bc.LIB_PATH), "tile": t, "ms": round(ms, 4),
                  "tflops": round(fl / ms / 1e9, 2), "fp64_frac": round(fl / ms / 1e9 / 37.2, 3),
                  "energy": float(ws[0].item())}))
