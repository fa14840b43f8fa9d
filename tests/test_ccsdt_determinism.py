"""Repeat-run determinism stress gate for the warp-specialised TMA CCSD(T) kernels (GPU).

The fused d1/d2 kernels (row a11) accumulate each t3 position in a fixed
order: per class, one owning thread adds its DMMA accumulator, and the classes run in
entry order.  Without a race, repeated launches on identical inputs are bitwise
identical.  A ring or flush race shows up as a few hundred t3 elements that differ
between runs.  The small parity tests never reached that state; this gate runs the
bench's configuration (tile 16, 8 blocks, all 9 variants of d1 then d2), the exact-24-cube
kernel (tile 24, 2 blocks) and the f4 energy kernels REPEATS times each.

Negative control: the tile-16 kernel built WITHOUT the generic->async
proxy fence before its ring-slot release failed this configuration in 183 of 200 runs
(128-1648 t3 values per run); with the fence 0 of 200.
"""
import pytest
import torch

import paper_conf_icpp_nelsonrbhhjn15_b200 as bc

pytestmark = pytest.mark.gpu

REPEATS = 40


def _ops(tile, dev, blocks):
    f64 = torch.float64
    base = [bc.fill(torch.empty(tile ** 6, dtype=f64, device=dev), 10 + 100 * b) for b in range(blocks)]
    ops = {f: ([bc.fill(torch.empty(tile ** 4, dtype=f64, device=dev), 20 + v + 50 * i) for v in range(9)],
               [bc.fill(torch.empty(tile ** 4, dtype=f64, device=dev), 40 + v + 50 * i) for v in range(9)])
           for i, f in enumerate(("d1", "d2"))}
    return base, ops


@pytest.mark.parametrize("tile,blocks", [(16, 8), (24, 2)])
def test_fused_repeat_bitwise(tile, blocks):
    dev = torch.device("cuda:0")
    ext = (tile,) * 7
    base, ops = _ops(tile, dev, blocks)
    first = None
    bad = []
    for r in range(REPEATS):
        t3 = [x.clone() for x in base]
        for f in ("d1", "d2"):
            for b in range(blocks):
                bc.ccsdt_fused(f, ext, t3[b], *ops[f])
        torch.cuda.synchronize()
        if first is None:
            first = t3
            assert all(not torch.equal(a, b) for a, b in zip(first, base)), "fused kernels left t3 unchanged"
            continue
        nd = sum(int((t3[b] != first[b]).sum().item()) for b in range(blocks))
        if nd:
            bad.append((r, nd))
    assert not bad, f"{len(bad)} of {REPEATS - 1} repeat runs differ from run 0 (run, #elements): {bad[:8]}"


@pytest.mark.parametrize("tile", [16, 24])
def test_triples_energy_repeat_bitwise(tile):
    """f4 (27 variants + energy epilogue; 16-cube and exact-24-cube TMA kernels): the
    energy of repeated launches is bitwise equal (fixed per-CTA unit order, fixed-order
    partial sums)."""
    dev = torch.device("cuda:0")
    f64 = torch.float64
    ext = (tile, tile, tile, 4, 4, 4, tile)
    H, P = tile, 4
    n = {"s1": (P * H, H * H * P * P), "d1": (tile * P * P * H, H * H * P * tile),
         "d2": (tile * P * H * H, tile * H * P * P)}
    fams = {}
    for i, f in enumerate(("s1", "d1", "d2")):
        fams[f] = ([bc.fill(torch.empty(n[f][0], dtype=f64, device=dev), 300 + 20 * i + v) for v in range(9)],
                   [bc.fill(torch.empty(n[f][1], dtype=f64, device=dev), 400 + 20 * i + v) for v in range(9)])
    eh = bc.fill(torch.empty(3 * H, dtype=f64, device=dev), 60, kind=bc.KIND_RANGE, lo=-2.0, hi=-0.5)
    ep = bc.fill(torch.empty(3 * P, dtype=f64, device=dev), 61, kind=bc.KIND_RANGE, lo=0.5, hi=2.0)
    vals = []
    for _ in range(REPEATS // 2):
        ws = torch.empty(bc.BC_CHECK_WS_DOUBLES, dtype=f64, device=dev)
        bc.ccsdt_triples_energy(ext, fams["s1"], fams["d1"], fams["d2"], eh, ep, ws=ws)
        vals.append(float(ws[0].item()))
    assert vals[0] != 0.0
    assert len(set(vals)) == 1, f"energies differ across repeats: {sorted(set(vals))[:4]}"
