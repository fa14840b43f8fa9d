"""Multi-GPU host logic on CPU: shard plan, and the world-size-2 path over gloo
(process group init, check-scalar SUM, max-over-ranks), with the oracle standing in for
the per-rank compute so no GPU is needed."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

from paper_conf_icpp_nelsonrbhhjn15_b200 import dist as bdist


@pytest.mark.parametrize("world", [1, 2, 3, 4, 7, 8])
@pytest.mark.parametrize("n", [0, 1, 5, 8, 262144, 1000003])
def test_shard_plan_partitions(n, world):
    ranges = [bdist.shard(n, r, world) for r in range(world)]
    assert ranges[0][0] == 0 and ranges[-1][1] == n
    for (a, b), (c, d) in zip(ranges, ranges[1:]):
        assert b == c and a <= b
    sizes = [b - a for a, b in ranges]
    assert max(sizes) - min(sizes) <= 1
    for u in ([0, n // 2, n - 1] if n else []):
        r = bdist.owner(u, n, world)
        a, b = ranges[r]
        assert a <= u < b


def test_weak_scaling_slices_are_the_global_batch():
    """Rank r generates global elements [r*N, (r+1)*N): concatenated = one global batch."""
    import synthetic as syn
    P1, N, G = 4, 5, 3
    parts = [syn.elements(syn.TID["U"], P1, np.arange(r * N, (r + 1) * N)) for r in range(G)]
    whole = syn.tensor(syn.TID["U"], (G * N, P1, P1, P1))
    assert np.array_equal(np.concatenate(parts), whole)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import oracle
    import synthetic as syn
    rk = bdist.init(backend="gloo")
    P1, Ntot = 5, 37
    a, b = bdist.shard(Ntot, rk.rank, rk.world)
    U = syn.elements(syn.TID["U"], P1, np.arange(a, b))
    A = syn.tensor(syn.TID["A"], (P1, P1))
    V = oracle.sumfact3d(A, A, A, U)
    chk = torch.tensor([float((V * V).sum())], dtype=torch.float64)
    bdist.all_reduce_sum_(chk)
    t = bdist.max_over_ranks(float(rk.rank + 1) * 1.5, torch.device("cpu"))
    bdist.barrier()
    q.put((rk.rank, float(chk.item()), t))
    bdist.finalize()


def test_gloo_world2_check_sum_and_max():
    import oracle
    import synthetic as syn
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    P1, Ntot = 5, 37
    U = syn.tensor(syn.TID["U"], (Ntot, P1, P1, P1))
    A = syn.tensor(syn.TID["A"], (P1, P1))
    V = oracle.sumfact3d(A, A, A, U)
    ref = float((V * V).sum())
    for rank, chk, t in res:
        assert abs(chk - ref) <= 1e-12 * ref
        assert t == 3.0
