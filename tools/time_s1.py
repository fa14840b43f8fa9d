"""Time the fused s1 kernel (9 variants, one full tile block) for a given build
(BARRACUDA_LIB); fraction of the HBM copy peak (t3 read + write)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t = int(os.environ.get("TILE", "16"))
ext = (t,) * 7
f64, dev = torch.float64, "cuda"
t3 = bc.fill(torch.empty(t ** 6, dtype=f64, device=dev), 10)
na, nb = bc.operand_sizes("s1", ext)
ops = ([bc.fill(torch.empty(na, dtype=f64, device=dev), 100 + v) for v in range(9)],
       [bc.fill(torch.empty(nb, dtype=f64, device=dev), 110 + v) for v in range(9)])
run = lambda: bc.ccsdt_fused("s1", ext, t3, *ops)  # noqa: E731
run(); torch.cuda.synchronize()
reps = 40 if t == 16 else 6
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); [run() for _ in range(reps)]; e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
by = 16.0 * t ** 6
print(json.dumps({"lib": os.path.basename(bc.LIB_PATH), "tile": t, "us": round(ms * 1e3, 2),
                  "gbs": round(by / ms / 1e6, 1), "hbm_frac": round(by / ms / 1e6 / 6539.2, 3)}))
