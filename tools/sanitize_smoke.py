"""Small invocations of every kernel family, for compute-sanitizer runs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
import synthetic as syn
dev = torch.device("cuda")
f = lambda shape, tid: bc.fill(torch.empty(shape, dtype=torch.float64, device=dev), tid)
# P1 = 8 and 16 take the DMMA spectral kernels; N = 7 the shared-memory-operator kernels,
# N = 130 the constant-bank-operator kernels
for P1, N in ((5, 7), (5, 130), (8, 7), (13, 7), (13, 130), (16, 7)):
    U = f((N, P1, P1, P1), 1); A = f((P1, P1), 2)
    bc.sumfact3d(A, A, A, U); bc.sumfact3d(A, A, A, U, check_ws=torch.empty(1024, dtype=torch.float64, device=dev))
    bc.sumfact2d(A, A, f((N + 2, P1, P1), 3))
    D = torch.from_numpy(syn.gll_derivative(P1 - 1)).to(dev)
    r = bc.local_grad3(D, U); bc.local_grad3_t(D, *r); bc.ax_e(D, U, f((N, 6, P1, P1, P1), 11))
    U32 = U.float(); bc.sumfact3d(A.float(), A.float(), A.float(), U32)
for ext in ((16,) * 7, (20, 20, 20, 4, 4, 4, 6), (3, 4, 5, 6, 2, 7, 3)):
    h1, h2, h3, p4, p5, p6, k = ext
    n3 = h1 * h2 * h3 * p4 * p5 * p6
    t3 = f((n3,), 10)
    for fam, (na, nb) in (("d1", (k * p4 * p5 * h1, h3 * h2 * p6 * k)), ("d2", (k * p4 * h1 * h2, k * h3 * p6 * p5)),
                          ("s1", (p4 * h1, h3 * h2 * p6 * p5))):
        xs = [f((na,), 20 + v) for v in range(9)]; ys = [f((nb,), 40 + v) for v in range(9)]
        bc.ccsdt(fam, 5, ext, t3, xs[4], ys[4]); bc.ccsdt_fused(fam, ext, t3, xs, ys)
    if h1 == h2 == h3 and h1 % 2 == 0 and h1 >= 12 and k % 2 == 0:
        tr = lambda na, nb: ([f((na,), 60 + v) for v in range(9)], [f((nb,), 70 + v) for v in range(9)])
        bc.ccsdt_triples_energy(ext, tr(p4 * h1, h3 * h2 * p6 * p5), tr(k * p4 * p5 * h1, h3 * h2 * p6 * k),
                                tr(k * p4 * h1 * h2, k * h3 * p6 * p5), f((3 * h1,), 60), f((3 * p4,), 61))
    bc.check_energy(ext, t3, f((h1 + h2 + h3,), 60), f((p4 + p5 + p6,), 61))
bc.check_sumsq(f((100000,), 1))
torch.cuda.synchronize()
print("sanitize smoke: done")
