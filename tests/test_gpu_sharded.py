"""Cell-ownership sharding (include/ggrid.h "cell-ownership sharding") on one GPU:
`world` processes share cuda:0, each holding a ggrid_shard-ed handle, exchanging over gloo
(host-staged all-to-all; NCCL is the same code path between GPUs).  Answers must equal the
oracle bit for bit, the remote masks must be selective, and a single-rank handle must answer
exactly as before."""
import os
import socket

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gg():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icde_li0qhdy18_b200 import build

    build.build()
    import paper_conf_icde_li0qhdy18_b200 as m

    return m


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg, routed, q_out):
    import torch
    import torch.distributed as dist

    import paper_conf_icde_li0qhdy18_b200 as gg
    from paper_conf_icde_li0qhdy18_b200 import dist as gdist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        scale, cs, n_obj, k, nq = cfg
        g = synth.table_ii_graph("NY", scale=scale)
        walk = synth.RandomWalk(g, n_obj, inject=True)
        grid = gg.GGrid(g, cs, max_objects=n_obj).shard(world, rank)
        hist = []
        for _ in range(3):
            u = walk.ticks(2)
            hist.append(u)
            grid.ingest(u)
        upd = np.concatenate(hist)
        q = synth.queries(g, nq)
        qt_all = torch.from_numpy(q.view(np.int32)).cuda()
        if routed:
            owner = grid.query_owner(qt_all, torch.empty(nq, dtype=torch.int32, device="cuda"))
            sel = (owner == rank).cpu().numpy()
        else:
            lo, hi = gdist.shard_range(nq, rank, world)
            sel = np.zeros(nq, bool)
            sel[lo:hi] = True
        mine = q[sel]
        qt = torch.from_numpy(mine.view(np.int32)).cuda().reshape(-1, 2)
        o, d, n_req = gdist.sharded_knn(grid, qt, k, world, rank, routed=routed)
        ro, rd = oracle.knn_from_updates(g, upd, mine, k)
        go = o.cpu().numpy().view(np.uint32)
        gd = d.cpu().numpy().view(np.uint32)
        bad = np.flatnonzero(~((go == ro).all(1) & (gd == rd).all(1)))
        st = grid.stats()
        q_out.put((rank, len(bad), len(mine), n_req, int(st["objects_written"])))
    finally:
        dist.destroy_process_group()


def _run(world, cfg, routed):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q_out = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, routed, q_out)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q_out.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
    return res


@pytest.mark.parametrize("world,routed", [(2, False), (3, True), (4, False)])
def test_sharded_knn_exact(gg, world, routed):
    res = _run(world, (0.05, 256, 2000, 10, 400), routed)
    assert all(bad == 0 for _, bad, _, _, _ in res), res
    n_q = sum(n for _, _, n, _, _ in res)
    n_req = sum(r for _, _, _, r, _ in res)
    assert n_q == 400
    assert 0 < n_req < (world - 1) * n_q, res  # exchanged, and selectively
    assert all(w > 0 for *_, w in res)  # every rank holds objects of its own cells


def test_sharded_large_k_and_sparse(gg):
    """k beyond the first level and few objects (big balls crossing many owners)."""
    res = _run(3, (0.05, 128, 150, 40, 200), False)
    assert all(bad == 0 for _, bad, _, _, _ in res), res


def test_shard_after_ingest_rejected(gg):
    g = synth.table_ii_graph("NY", scale=0.02)
    grid = gg.GGrid(g, 64, max_objects=10)
    grid.ingest(np.array([[1, 0, 0, 5]], np.uint32))
    with pytest.raises(gg.GGridError):
        grid.shard(2, 0)
    with pytest.raises(gg.GGridError):
        gg.GGrid(g, 64).shard(2, 2)
    grid.close()
