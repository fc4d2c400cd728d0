"""Multi-GPU driver: one process per GPU, lookups sharded by index range, grid replicated.

SURVEY.md §8e: lookups are independent (counter-based RNG: lookup i depends only on
(seed, i)), so rank r of R owns an index range and the data path has no collective.
The only exchange is the verification reduction -- NCCL all_reduce SUM of
{hash, lookups, pairs} and MAX of the device time -- plus a one-off MIN/MAX of the
grid checksum that proves every replica is identical.  torch.distributed is the
plumbing; the backend is whatever the process group was created with (nccl on the
B200 box, gloo in the CPU tests).
"""
from __future__ import annotations

import os
from dataclasses import dataclass

import torch
import torch.distributed as dist


@dataclass
class Rank:
    rank: int = 0
    world: int = 1
    local_rank: int = 0

    @property
    def distributed(self) -> bool:
        return self.world > 1


def local_device(local: int) -> int:
    """The GPU of local rank `local`: one per GPU; with more ranks than visible GPUs (a gloo
    test of the N > 1 path on a 1-GPU box) ranks share them round-robin."""
    n = torch.cuda.device_count()
    return local % n if n > 0 else 0


def init(backend: str | None = None) -> Rank:
    """Join the process group torchrun describes (RANK/WORLD_SIZE/LOCAL_RANK/MASTER_*).
    backend: "nccl" (default with CUDA: NVLink / NVSwitch on the B200 node) or "gloo"."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and not dist.is_initialized():
        if backend is None:
            backend = "nccl" if torch.cuda.is_available() else "gloo"
        if backend == "nccl":
            if torch.cuda.device_count() < world:
                raise RuntimeError(f"nccl needs one GPU per rank: {world} ranks, "
                                   f"{torch.cuda.device_count()} GPUs (XS_DIST_BACKEND=gloo shares them)")
            torch.cuda.set_device(local)
            dist.init_process_group(backend, device_id=torch.device("cuda", local))
        else:
            if torch.cuda.is_available():
                torch.cuda.set_device(local_device(local))
            dist.init_process_group(backend)
    elif torch.cuda.is_available():
        torch.cuda.set_device(local_device(local))
    return Rank(rank, world, local)


def backend_name() -> str:
    return dist.get_backend() if dist.is_initialized() else "none (1 process)"


def shard(total: int, rank: int, world: int) -> tuple[int, int]:
    """Strong-scaling split of [0, total): rank r gets [floor(r*T/R), floor((r+1)*T/R))."""
    a = total * rank // world
    b = total * (rank + 1) // world
    return a, b - a


def weak_range(per_rank: int, rank: int) -> tuple[int, int]:
    """Weak-scaling split: every rank owns its own per_rank lookups."""
    return per_rank * rank, per_rank


def _device(backend_device=None):
    if backend_device is not None:
        return backend_device
    if dist.is_initialized() and dist.get_backend() == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def reduce_stats(hash_: int, lookups: int, pairs: int, device_ms: float, device=None):
    """(hash, lookups, pairs) SUM and device_ms MAX over ranks; identity without a group."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return hash_, lookups, pairs, device_ms
    dev = _device(device)
    counts = torch.tensor([hash_, lookups, pairs], dtype=torch.int64, device=dev)
    ms = torch.tensor([device_ms], dtype=torch.float64, device=dev)
    dist.all_reduce(counts, op=dist.ReduceOp.SUM)
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    c = counts.tolist()
    return int(c[0]), int(c[1]), int(c[2]), float(ms.item())


def replicas_identical(checksum: int, device=None) -> bool:
    """MIN == MAX of the grid checksum over ranks."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return True
    dev = _device(device)
    v = checksum - (1 << 64) if checksum >= (1 << 63) else checksum  # as int64
    lo = torch.tensor([v], dtype=torch.int64, device=dev)
    hi = lo.clone()
    dist.all_reduce(lo, op=dist.ReduceOp.MIN)
    dist.all_reduce(hi, op=dist.ReduceOp.MAX)
    return int(lo.item()) == int(hi.item())


def sum_over_ranks(x: int, device=None) -> int:
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return x
    t = torch.tensor([x], dtype=torch.int64, device=_device(device))
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return int(t.item())


def min_over_ranks(x: int, device=None) -> int:
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return x
    t = torch.tensor([x], dtype=torch.int64, device=_device(device))
    dist.all_reduce(t, op=dist.ReduceOp.MIN)
    return int(t.item())


def max_over_ranks(x: float, device=None) -> float:
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=_device(device))
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier():
    if dist.is_initialized() and dist.get_world_size() > 1:
        if dist.get_backend() == "nccl":
            dist.barrier(device_ids=[torch.cuda.current_device()])
        else:
            dist.barrier()


def finalize():
    if dist.is_initialized():
        dist.destroy_process_group()
