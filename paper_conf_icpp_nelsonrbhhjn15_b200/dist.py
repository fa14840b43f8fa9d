"""Multi-GPU plumbing: one process per GPU, torch.distributed for the
process group, contiguous shard plans, and the only collectives the path has — scalar
check reductions and the max-over-ranks of timings.  Elements and CCSD(T) tile blocks are
independent, so no data crosses between GPUs.
"""
from __future__ import annotations

import os
from dataclasses import dataclass

import torch
import torch.distributed as dist


@dataclass(frozen=True)
class Rank:
    rank: int
    world: int
    local_rank: int
    device: torch.device


def init(backend: str | None = None) -> Rank:
    """Read RANK / WORLD_SIZE / LOCAL_RANK (torchrun); init the process group if world > 1.
    backend defaults to nccl when CUDA is available, else gloo (BC_DIST_BACKEND overrides;
    with more ranks than GPUs — a test configuration — ranks share GPUs modulo the count
    and must use gloo, since NCCL needs one GPU per rank)."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    backend = backend or os.environ.get("BC_DIST_BACKEND")
    if torch.cuda.is_available():
        dev_index = local % torch.cuda.device_count()
        torch.cuda.set_device(dev_index)
        device = torch.device("cuda", dev_index)
    else:
        device = torch.device("cpu")
    if world > 1 and not dist.is_initialized():
        if backend is None:
            backend = "nccl" if device.type == "cuda" else "gloo"
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group(backend=backend, rank=rank, world_size=world,
                                device_id=device if backend == "nccl" else None)
    return Rank(rank, world, local, device)


def shard(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous range [floor(r n / G), floor((r+1) n / G)) of n units owned by rank r."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return (rank * n) // world, ((rank + 1) * n) // world


def owner(unit: int, n: int, world: int) -> int:
    """Rank owning unit `unit` under shard(); inverse of the plan."""
    if not 0 <= unit < n:
        raise ValueError("unit out of range")
    r = (unit * world) // n
    while shard(n, r, world)[1] <= unit:
        r += 1
    while shard(n, r, world)[0] > unit:
        r -= 1
    return r


def barrier() -> None:
    if dist.is_initialized():
        if dist.get_backend() == "nccl":
            dist.barrier(device_ids=[torch.cuda.current_device()])
        else:
            dist.barrier()


def _coll_device(device: torch.device) -> torch.device:
    # gloo reduces host tensors; NCCL device tensors
    return device if dist.get_backend() == "nccl" else torch.device("cpu")


def all_reduce_sum_(t: torch.Tensor) -> torch.Tensor:
    """In-place SUM of a (small) check tensor over ranks; identity when world == 1."""
    if dist.is_initialized() and dist.get_world_size() > 1:
        cd = _coll_device(t.device)
        if cd == t.device:
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
        else:
            h = t.to(cd)
            dist.all_reduce(h, op=dist.ReduceOp.SUM)
            t.copy_(h)
    return t


def max_over_ranks(x: float, device: torch.device) -> float:
    if dist.is_initialized() and dist.get_world_size() > 1:
        t = torch.tensor([x], dtype=torch.float64, device=_coll_device(device))
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    return x


def sum_over_ranks(x: float, device: torch.device) -> float:
    """SUM of a host scalar over ranks (e.g. the flops each rank's shard performed)."""
    if dist.is_initialized() and dist.get_world_size() > 1:
        t = torch.tensor([x], dtype=torch.float64, device=_coll_device(device))
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())
    return x


def finalize() -> None:
    if dist.is_initialized():
        dist.destroy_process_group()
