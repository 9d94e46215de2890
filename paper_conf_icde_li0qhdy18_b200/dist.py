"""Multi-GPU plumbing over torch.distributed.

One process per GPU.  The update stream is broadcast from the rank that receives it (NCCL over
NVLink on GPUs, gloo in CPU tests).  Two layouts:
  * cell-ownership sharding (default): each rank's handle keeps the logs of its
    own cells only; queries are answered with one request/reply exchange (sharded_knn below);
  * replicas: every rank holds the whole index and answers its own contiguous share of the
    queries with no collective in the query phase.
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


# ---- cell-ownership sharding (include/ggrid.h "cell-ownership sharding") --------
#
# Each rank's handle is ggrid_shard(world, rank)-ed: it owns a contiguous Z-order range of cells
# and keeps logs/lists only for them; every rank ingests the whole update stream (object table
# replicated).  A batch of queries is answered exactly with one request/reply exchange:
#   route    each query to the owner of its cell                          (all-to-all)
#   primary  owner: k nearest of its own objects + mask of other ranks' cells its search entered
#   request  (query, bound = owner's k-th distance) to every masked rank  (all-to-all)
#   reply    each such rank: its own objects within the bound, <= k       (all-to-all)
#   merge    owner: k-way merge (ggrid_merge_topk)
#   return   answers to the rank the query came from                      (all-to-all)
# The packing below is argument marshalling (index/concatenate); every per-query computation
# (search, bound, mask, merge) runs in libggrid.so.

def _a2a(inp, in_counts, world):
    """all_to_all_single of the rows of `inp` (grouped by destination, in_counts rows each);
    returns (received rows grouped by source, counts per source).  gloo (CPU tests / one-GPU
    multi-process runs) exchanges through host memory, NCCL directly between GPUs."""
    import torch
    import torch.distributed as dist

    via_host = dist.get_backend() == "gloo" and inp.is_cuda
    ic = torch.as_tensor(in_counts, dtype=torch.int64)
    oc = torch.empty_like(ic)
    if via_host or not inp.is_cuda:
        dist.all_to_all_single(oc, ic)
    else:
        ic_d = ic.to(inp.device)
        oc_d = torch.empty_like(ic_d)
        dist.all_to_all_single(oc_d, ic_d)
        oc = oc_d.cpu()
    cols = inp.shape[1]
    src = inp.cpu() if via_host else inp
    out = src.new_empty((int(oc.sum()), cols))
    dist.all_to_all_single(out, src.contiguous(), [int(x) for x in oc], [int(x) for x in ic])
    if via_host:
        out = out.to(inp.device)
    return out, [int(x) for x in oc]


def _group_by(dest, world):
    """Stable order grouping items by destination rank, and the per-rank counts."""
    import torch

    order = torch.argsort(dest.to(torch.int64), stable=True)
    counts = torch.bincount(dest.to(torch.int64), minlength=world).cpu().tolist()
    return order, counts


def sharded_knn(grid, queries, k: int, world: int, rank: int, routed: bool = False):
    """Exact kNN of this rank's queries ((n, 2) int32 CUDA tensor) on a sharded index.
    Library calls are ordered after torch's current stream by the binding (ggrid_wait_stream),
    so the torch ops and collectives that produce their inputs need no host synchronisation.
    routed=True: every query is already at the owner of its cell (skips route/return).
    Returns (obj, dist) int32 CUDA tensors (n, k), and the number of remote requests sent."""
    import torch

    dev = queries.device
    n = int(queries.shape[0])
    i32 = torch.int32

    idx = torch.arange(n, dtype=i32, device=dev)
    if routed:
        mine, src_counts = torch.cat([queries, idx[:, None]], 1), None
    else:
        owner = torch.empty(n, dtype=i32, device=dev)
        grid.query_owner(queries, owner)
        order, counts = _group_by(owner, world)
        mine, src_counts = _a2a(torch.cat([queries, idx[:, None]], 1)[order], counts, world)
    m = int(mine.shape[0])
    q_m = mine[:, :2].contiguous()
    own_o = torch.empty((m, k), dtype=i32, device=dev)
    own_d = torch.empty((m, k), dtype=i32, device=dev)
    mask = torch.empty(m, dtype=torch.int64, device=dev)
    grid.knn_ex(q_m, k, None, own_o, own_d, mask)
    # requests: (edge, offset, bound, local row) to every rank in the mask
    bits = ((mask[:, None] >> torch.arange(world, device=dev, dtype=torch.int64)[None, :]) & 1).bool()
    qi, tgt = torch.nonzero(bits, as_tuple=True)
    req = torch.cat([q_m[qi], own_d[qi, k - 1:k], qi.to(i32)[:, None]], 1)
    order_r, counts_r = _group_by(tgt, world)
    got, got_counts = _a2a(req[order_r], counts_r, world)
    rep_o = torch.empty((int(got.shape[0]), k), dtype=i32, device=dev)
    rep_d = torch.empty_like(rep_o)
    got_q, got_b = got[:, :2].contiguous(), got[:, 2].contiguous()
    grid.knn_ex(got_q, k, got_b, rep_o, rep_d)
    replies, _ = _a2a(torch.cat([rep_o, rep_d, got[:, 3:4], torch.full_like(got[:, 3:4], rank)], 1),
                      got_counts, world)
    # dense [world][m][k] lists: own list at slot `rank`, the reply of rank t at slot t
    lo = torch.full((world, m, k), -1, dtype=i32, device=dev)
    ld = torch.full((world, m, k), -1, dtype=i32, device=dev)
    lo[rank] = own_o
    ld[rank] = own_d
    if replies.shape[0]:
        r_q = replies[:, 2 * k].long()
        r_t = replies[:, 2 * k + 1].long()
        lo[r_t, r_q] = replies[:, :k]
        ld[r_t, r_q] = replies[:, k:2 * k]
    fo = torch.empty((m, k), dtype=i32, device=dev)
    fd = torch.empty((m, k), dtype=i32, device=dev)
    grid.merge_topk(lo, ld, fo, fd)
    if routed:
        return fo, fd, int(req.shape[0])
    # answers back to the ranks the queries came from, into their original rows
    ans, _ = _a2a(torch.cat([fo, fd, mine[:, 2:3]], 1), src_counts, world)
    out_o = torch.empty((n, k), dtype=i32, device=dev)
    out_d = torch.empty((n, k), dtype=i32, device=dev)
    rows = ans[:, 2 * k].long()
    out_o[rows] = ans[:, :k]
    out_d[rows] = ans[:, k:2 * k]
    return out_o, out_d, int(req.shape[0])
