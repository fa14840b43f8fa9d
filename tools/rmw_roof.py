"""Achievable HBM bandwidth of an in-place read-modify-write stream (torch add_ / mul_)
vs an out-of-place copy, at the CCSD(T) t3 sizes (tile 16: 134 MB, tile 24: 1.53 GB) and
1 GiB — the practical ceiling for the HBM-bound t3 += X kernels.  Prints one JSON line."""
import json
import torch

res = {}
for name, n in (("t3_tile16", 16 ** 6), ("t3_tile24", 24 ** 6), ("1GiB", 2 ** 27)):
    x = torch.randn(n, dtype=torch.float64, device="cuda")
    y = torch.empty_like(x)
    flush = torch.empty(256 * 2 ** 20 // 8, dtype=torch.float64, device="cuda")
    for kind, fn in (("rmw_add", lambda: x.add_(1.0)), ("copy", lambda: y.copy_(x))):
        for _ in range(3):
            fn()
        ts = []
        for _ in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = sorted(ts)[len(ts) // 2]
        res[f"{name}_{kind}_gbs"] = round(2 * n * 8 / ms / 1e6, 1)
    del x, y
print(json.dumps(res))
