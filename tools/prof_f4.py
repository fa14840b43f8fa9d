"""Launch the f4 triples+energy kernel a few times (TILE, default 24; particle extent 2) —
for ncu under gpurun."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t = int(os.environ.get("TILE", "24")); pp = int(os.environ.get("PP", "4"))
ext = (t, t, t, pp, pp, pp, t)
dev = "cuda"
def ops(base, n):
    return [bc.fill(torch.empty(n, dtype=torch.float64, device=dev), base + v) for v in range(9)]
s1 = (ops(50, pp * t), ops(70, t * t * pp * pp))
d1 = (ops(20, t * pp * pp * t), ops(40, t * t * pp * t))
d2 = (ops(200020, t * pp * t * t), ops(200040, t * t * pp * pp))
eh = bc.fill(torch.empty(3 * t, dtype=torch.float64, device=dev), 60, kind=bc.KIND_RANGE, lo=-2.0, hi=-0.5)
ep = bc.fill(torch.empty(3 * pp, dtype=torch.float64, device=dev), 61, kind=bc.KIND_RANGE, lo=0.5, hi=2.0)
for _ in range(3):
    bc.ccsdt_triples_energy(ext, s1, d1, d2, eh, ep)
torch.cuda.synchronize()
print("ok")
