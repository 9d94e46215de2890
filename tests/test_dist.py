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


# ---- cell-ownership sharding protocol (dist.sharded_knn), host logic on CPU ---------------------
class _FakeShard:
    """CPU stand-in for one rank's sharded handle: the oracle over the objects whose latest
    location lies in this rank's cells (cells = vertex-id ranges here).  Its remote mask names
    every other rank (the widest mask the protocol must tolerate); the real mask is the GPU
    test's subject."""

    def __init__(self, g, upd, world, rank, n_cells=16):
        import oracle

        self.g, self.world, self.rank = g, world, rank
        self.n_cells, V = n_cells, g["n_vertices"]
        ids, e, o = oracle.snapshot_objects(upd)
        own = self._owner_of_edge(e) == rank
        self.ids, self.e, self.o = ids[own], e[own], o[own]

    def _owner_of_edge(self, e):
        cell = self.g["src"][np.asarray(e, np.int64)].astype(np.int64) * self.n_cells // self.g["n_vertices"]
        return cell * self.world // self.n_cells

    def query_owner(self, q, out):
        out[:] = torch.from_numpy(self._owner_of_edge(q[:, 0].numpy().view(np.uint32)).astype(np.int32))

    def knn_ex(self, q, k, bound, out_o, out_d, out_mask=None):
        import oracle

        qq = q.numpy().view(np.uint32)
        o, d = oracle.knn(self.g, self.ids, self.e, self.o, qq, k)
        if bound is not None:
            b = bound.numpy().view(np.uint32)[:, None]
            far = d > b
            o[far] = 0xFFFFFFFF
            d[far] = 0xFFFFFFFF
        out_o[:] = torch.from_numpy(o.view(np.int32))
        out_d[:] = torch.from_numpy(d.view(np.int32))
        if out_mask is not None:
            out_mask[:] = sum(1 << t for t in range(self.world) if t != self.rank)

    def merge_topk(self, lo, ld, fo, fd):
        L, m, k = lo.shape
        o = lo.numpy().view(np.uint32).transpose(1, 0, 2).reshape(m, L * k)
        d = ld.numpy().view(np.uint32).transpose(1, 0, 2).reshape(m, L * k)
        key = (d.astype(np.uint64) << np.uint64(32)) | o.astype(np.uint64)
        key = np.sort(key, axis=1)[:, :k]
        fo[:] = torch.from_numpy((key & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32))
        fd[:] = torch.from_numpy((key >> np.uint64(32)).astype(np.uint32).view(np.int32))


def _shard_worker(rank, world, port, routed, q_out):
    import oracle
    import synth

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = synth.table_ii_graph("NY", scale=0.02)
        upd = synth.RandomWalk(g, 400, inject=True).ticks(3)
        grid = _FakeShard(g, upd, world, rank)
        q = synth.queries(g, 90 + world)
        lo, hi = gdist.shard_range(len(q), rank, world)
        mine = q[lo:hi]
        if routed:  # every rank takes the queries it owns
            own = grid._owner_of_edge(q[:, 0]) == rank
            mine = q[own]
        qt = torch.from_numpy(mine.astype(np.uint32).view(np.int32)).reshape(-1, 2)
        o, d, n_req = gdist.sharded_knn(grid, qt, 6, world, rank, routed=routed)
        ro, rd = oracle.knn_from_updates(g, upd, mine, 6)
        ok = np.array_equal(o.numpy().view(np.uint32), ro) and np.array_equal(d.numpy().view(np.uint32), rd)
        q_out.put((rank, bool(ok), n_req))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,routed", [(2, False), (3, False), (2, True)])
def test_sharded_protocol_exact(world, routed):
    """Route -> owner search -> bounded remote requests -> replies -> merge -> return, over
    gloo with `world` CPU processes, equals the single-process oracle answer row for row."""
    ctx = mp.get_context("spawn")
    q_out = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, world, port, routed, q_out)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q_out.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok, _ in res), res
    assert sum(n for _, _, n in res) > 0  # the exchange was exercised
