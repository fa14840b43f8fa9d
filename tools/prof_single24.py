"""Launch single-variant d1 / d2 at tile 24 a few times (for ncu under gpurun)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_nelsonrbhhjn15_b200 as bc
t = 24; ext = (t,) * 7
t3 = bc.fill(torch.empty(t ** 6, dtype=torch.float64, device="cuda"), 10)
t2 = bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 21)
v2 = bc.fill(torch.empty(t ** 4, dtype=torch.float64, device="cuda"), 41)
for _ in range(3):
    bc.ccsdt("d1", 1, ext, t3, t2, v2)
    bc.ccsdt("d2", 2, ext, t3, t2, v2)
torch.cuda.synchronize()
