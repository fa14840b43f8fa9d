"""Time the spectral kernels for a given libbarracuda build (BARRACUDA_LIB=...).
Usage: python tools/sweep_spectral.py [p ...]   -> one line per (kernel, p)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_nelsonrbhhjn15_b200 as bc  # noqa: E402
import synthetic as syn  # noqa: E402

HBM = 6539.2


def timeit(fn, reps=10):
    fn(); fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


ps = [int(x) for x in sys.argv[1:]] or [12]
for p in ps:
    P1 = p + 1
    N = int(os.environ.get("N", str((262144 * 13 ** 3) // P1 ** 3)))
    U = torch.empty((N, P1, P1, P1), dtype=torch.float64, device="cuda")
    bc.fill(U, 1)
    A = bc.fill(torch.empty((P1, P1), dtype=torch.float64, device="cuda"), 2)
    D = torch.from_numpy(syn.gll_derivative(p)).cuda()
    V = torch.empty_like(U)
    outs = tuple(torch.empty_like(U) for _ in range(3))
    U2, V2 = U.view(-1, P1, P1), V.view(-1, P1, P1)
    res = {}
    for name, fn, by, fl in (
        ("local_grad3", lambda: bc.local_grad3(D, U, out=outs), 32 * P1 ** 3 * N, 6 * P1 ** 4 * N),
        ("sumfact3d", lambda: bc.sumfact3d(A, A, A, U, out=V), 16 * P1 ** 3 * N, 6 * P1 ** 4 * N),
        ("sumfact2d", lambda: bc.sumfact2d(A, A, U2, out=V2), 16 * P1 ** 3 * N, 4 * P1 ** 3 * N * P1),
        ("local_grad3_t", lambda: bc.local_grad3_t(D, *outs, out=V), 32 * P1 ** 3 * N, 6 * P1 ** 4 * N + 2 * P1 ** 3 * N),
        ("ax_e", "ax_e", 64 * P1 ** 3 * (N // 4), 12 * P1 ** 4 * (N // 4) + 17 * P1 ** 3 * (N // 4)),
    ):
        if os.environ.get("SWEEP_ONLY") and name not in os.environ["SWEEP_ONLY"].split(","):
            continue
        if fn == "ax_e":  # N/4 elements: G is 6 fields
            Na = N // 4
            G = bc.fill(torch.empty((Na, 6, P1, P1, P1), dtype=torch.float64, device="cuda"), 11)
            Ua, Wa = U[:Na], V[:Na]
            fn = lambda: bc.ax_e(D, Ua, G, out=Wa)  # noqa: E731
        ms = timeit(fn)
        res[name] = {"ms": round(ms, 4), "hbm_frac": round(by / ms / 1e6 / HBM, 3), "tflops": round(fl / ms / 1e9, 2)}
    print(json.dumps({"lib": os.path.basename(bc.LIB_PATH), "p": p, "N": N, **res}), flush=True)
    del U, V, outs
    torch.cuda.empty_cache()
