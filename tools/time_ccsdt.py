"""Time the fused CCSD(T) kernels (tile 16, 8 blocks) for a given build (BARRACUDA_LIB)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t = int(os.environ.get("TILE", "16")); nb = int(os.environ.get("BLOCKS", "8"))
ext = (t,) * 7
t3 = [bc.fill(torch.empty(t ** 6, dtype=torch.float64, device="cuda"), 10 + 100 * b) for b in range(nb)]
ops = {f: ([bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 20 + v) for v in range(9)],
           [bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 40 + v) for v in range(9)]) for f in ("d1", "d2")}
res = {"lib": os.path.basename(bc.LIB_PATH), "tile": t}
for f in ("d1", "d2"):
    run = lambda: [bc.ccsdt_fused(f, ext, t3[b], *ops[f]) for b in range(nb)]
    run(); run(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); [run() for _ in range(5)]; e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    res[f] = {"ms": round(ms, 3), "tflops": round(nb * 18 * t ** 7 / ms / 1e9, 2), "fp64_frac": round(nb * 18 * t ** 7 / ms / 1e9 / 37.2, 3)}
print(json.dumps(res))
