"""G-invariance of the sharded step: with the global batch split over G
ranks by dist.shard() (bench --scaling strong), every element's and every CCSD(T)
block's outputs are bitwise identical for G = 1, 2, 4, and the check scalars agree to
1e-12.  Inputs are keyed by global index (synthetic / bc_fill) and the kernels' per-unit
arithmetic does not depend on the grid (barracuda.h: results are deterministic), so only
the reduction order of the check scalars may change with G.

Runs G processes sharing the one GPU over gloo (NCCL needs one GPU per rank)."""
import os
import socket

import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

P, N_ELEM, BLOCKS, TILE = 5, 1001, 3, 16


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _hash_rows(x: torch.Tensor, n: int) -> torch.Tensor:
    """Exact per-row hash of fp64 bits: sum_j bits[j] * (2j+1) * phi (int64, wrapping)."""
    b = x.contiguous().view(torch.int64).reshape(n, -1)
    w = (torch.arange(b.shape[1], device=b.device, dtype=torch.int64) * 2 + 1) * 0x9E3779B97F4A7C1
    return (b * w).sum(dim=1).cpu().tolist()  # plain ints: tensors in a queue die with the sender


def _worker(rank, world, port, q):
    try:
        _work(rank, world, port, q)
    except BaseException:  # report instead of dying silently (the parent reads the queue)
        import traceback
        q.put({"rank": rank, "error": traceback.format_exc()})
        raise


def _work(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank), BC_DIST_BACKEND="gloo")
    from paper_conf_icpp_nelsonrbhhjn15_b200 import dist as bdist
    from paper_conf_icpp_nelsonrbhhjn15_b200.workload import Step, StepConfig
    rk = bdist.init()
    st = Step(StepConfig(p=P, n_elem=N_ELEM, tile=TILE, blocks=BLOCKS), rk.rank, rk.world, rk.device,
              scaling="strong")
    chk = st.run()
    torch.cuda.synchronize()
    n = st.n
    out = {"rank": rk.rank, "e0": st.e0, "b0": st.b0, "checks": chk.cpu().tolist()}
    if n:
        out["spectral"] = {nm: _hash_rows(getattr(st, nm), n) for nm in ("ur", "us", "ut", "V", "V2")}
    out["t3"] = [_hash_rows(t, 1) for t in st.t3]
    q.put(out)
    bdist.barrier()
    bdist.finalize()


def _run(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda d: d["rank"])
    errs = [r["error"] for r in res if "error" in r]
    assert not errs, errs[0]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    spectral = {nm: torch.tensor([h for r in res if "spectral" in r for h in r["spectral"][nm]])
                for nm in ("ur", "us", "ut", "V", "V2")}
    t3 = torch.tensor([h for r in res for blk in r["t3"] for h in blk])
    return spectral, t3, res[0]["checks"], [(r["e0"], r["b0"]) for r in res]


def test_outputs_bitwise_equal_for_G_1_2_4():
    ref_s, ref_t3, ref_chk, _ = _run(1)
    assert ref_s["ur"].numel() == N_ELEM and ref_t3.numel() == BLOCKS
    for world in (2, 4):
        s, t3, chk, starts = _run(world)
        assert [a for a, _ in starts] == [(r * N_ELEM) // world for r in range(world)]
        for nm in ref_s:
            nd = int((s[nm] != ref_s[nm]).sum())
            assert nd == 0, f"G={world}: {nd} elements of {nm} differ from G=1"
        assert torch.equal(t3, ref_t3), f"G={world}: t3 blocks differ from G=1"
        for a, b in zip(chk, ref_chk):
            assert abs(a - b) <= 1e-12 * abs(b), (world, chk, ref_chk)
