"""Launch the CCSD(T) streaming kernels a few times (tile 16): s1 fused (9 variants) and
d1 / d2 single variant — for ncu (-k regex:s1_stream|sv16) under gpurun."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t = int(os.environ.get("TILE", "16"))
ext = (t,) * 7
t3 = bc.fill(torch.empty(t ** 6, dtype=torch.float64, device="cuda"), 10)
t2 = [bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 20 + v) for v in range(9)]
v2 = [bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 40 + v) for v in range(9)]
t1 = [bc.fill(torch.empty(t * t, dtype=torch.float64, device="cuda"), 50 + v) for v in range(9)]
for _ in range(3):
    bc.ccsdt_fused("s1", ext, t3, t1, v2)
    bc.ccsdt("d1", 1, ext, t3, t2[0], v2[0])
    bc.ccsdt("d2", 3, ext, t3, t2[2], v2[2])
torch.cuda.synchronize()
