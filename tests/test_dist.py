"""World-size-2 gloo tests of the multi-GPU host logic, on CPU.

The GPU kernels cannot run here; what is checked is the orchestration the GPU path relies on:
the update batch broadcast reaches every replica bit-identically, query shards tile the batch
exactly once, the per-rank answers (computed here by the oracle, as a stand-in for each rank's
replica) reassemble into the single-process answer, and timings reduce to the max over ranks.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icde_li0qhdy18_b200 import dist as gdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q_out):
    import oracle
    import synth

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = synth.table_ii_graph("NY", scale=0.02)
        if rank == 0:
            upd = synth.RandomWalk(g, 300, inject=True).ticks(4)
            t = torch.from_numpy(upd.astype(np.int64))
        else:
            t = torch.zeros((1200, 4), dtype=torch.int64)
        gdist.broadcast_updates(t, src=0)
        upd = t.numpy().astype(np.uint32)
        q = synth.queries(g, 101)  # odd size: uneven shards
        lo, hi = gdist.shard_range(len(q), rank, world)
        o, d = oracle.knn_from_updates(g, upd, q[lo:hi], 5)
        allo = gdist.gather_rows(o, world)
        alld = gdist.gather_rows(d, world)
        slow = gdist.max_over_ranks(float(rank + 1))
        if rank == 0:
            ro, rd = oracle.knn_from_updates(g, synth.RandomWalk(g, 300, inject=True).ticks(4), q, 5)
            q_out.put((bool(np.array_equal(allo, ro) and np.array_equal(alld, rd)), slow))
    finally:
        dist.destroy_process_group()


def test_shard_range_tiles_exactly():
    for n in (0, 1, 7, 100, 101, 65536):
        for world in (1, 2, 3, 8):
            seen = []
            for r in range(world):
                lo, hi = gdist.shard_range(n, r, world)
                seen += list(range(lo, hi))
            assert seen == list(range(n))


def test_gloo_world2_broadcast_shard_gather():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs)
    ok, slow = q.get(timeout=5)
    assert ok
    assert slow == 2.0
