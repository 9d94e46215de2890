"""Multi-GPU plumbing over torch.distributed.

One process per GPU.  Every rank holds a full replica of the index; the update stream is
broadcast from the rank that receives it (NCCL over NVLink on GPUs, gloo in CPU tests) and
query batches are sharded into contiguous ranges, so the query phase needs no collective.
Only host-side orchestration lives here; all per-query and per-update work runs in
libggrid.so on each rank's GPU.
"""
from __future__ import annotations

import os


def env_rank():
    """(world, rank, local_rank) from the torchrun environment (1, 0, 0 when absent)."""
    return (int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
            int(os.environ.get("LOCAL_RANK", "0")))


def shard_range(n: int, rank: int, world: int):
    """Contiguous [lo, hi) share of n items for `rank`; the shares tile [0, n) exactly."""
    base, extra = divmod(n, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def broadcast_updates(t, src: int = 0):
    """Fan one update batch out to every replica (in place)."""
    import torch.distributed as dist

    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.broadcast(t, src)
    return t


def max_over_ranks(x: float, device=None) -> float:
    """Max of a per-rank scalar (timings are reported as the slowest rank)."""
    import torch
    import torch.distributed as dist

    if not (dist.is_initialized() and dist.get_world_size() > 1):
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_rows(arr, world: int):
    """Concatenate per-rank row blocks (numpy) on every rank, in rank order."""
    import numpy as np
    import torch
    import torch.distributed as dist

    if world == 1:
        return arr
    objs = [None] * world
    dist.all_gather_object(objs, arr)
    return np.concatenate(objs)
