"""Single-variant CCSD(T) tile-16 kernels side by side (env switches of run_ccsdt):
bulk-streamed sv16b (default), register-streamed sv16 (BC_SV16_REG), TMA cube kernel
(BC_NO_SV16); and s1 fused streaming vs the cube kernel (BC_NO_S1STREAM).
Back-to-back calls between CUDA events (host overhead overlapped)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
HBM = 6541.8
t = int(os.environ.get("TILE", "16")); ext = (t,) * 7; n3 = t ** 6
t3 = bc.fill(torch.empty(n3, dtype=torch.float64, device="cuda"), 10)
t2 = [bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 20 + v) for v in range(9)]
v2 = [bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 40 + v) for v in range(9)]
t1 = [bc.fill(torch.empty(t * t, dtype=torch.float64, device="cuda"), 50 + v) for v in range(9)]
flush = torch.empty(2 ** 25, dtype=torch.float64, device="cuda")
def timeit(fn, inner=20, reps=7):
    fn(); fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(inner):
            fn()
        e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / inner)
    return sorted(ts)[len(ts) // 2]
res = {"tile": t}
for env in ("", "BC_SV16_BULK", "BC_NO_SV16"):
    for k in ("BC_SV16_BULK", "BC_NO_SV16"):
        os.environ.pop(k, None)
    if env:
        os.environ[env] = "1"
    for f, v in (("d1", 1), ("d1", 3), ("d2", 1), ("d2", 2)):
        ms = timeit(lambda: bc.ccsdt(f, v, ext, t3, t2[v - 1], v2[v - 1]))
        res[f"{env or 'default'}_{f}v{v}"] = {"us": round(ms * 1e3, 1), "hbm_frac": round((16 * n3 + 16 * t ** 4) / ms / 1e6 / HBM, 3)}
for env in ("", "BC_NO_S1STREAM"):
    os.environ.pop("BC_NO_S1STREAM", None)
    if env:
        os.environ[env] = "1"
    ms = timeit(lambda: bc.ccsdt_fused("s1", ext, t3, t1, v2))
    res[f"{env or 'default'}_s1fused"] = {"us": round(ms * 1e3, 1), "hbm_frac": round((16 * n3) / ms / 1e6 / HBM, 3)}
print(json.dumps(res))
