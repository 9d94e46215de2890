"""Multi-GPU behind the C ABI (include/ggrid.h "multi-GPU") -- -m gpu.

One logical index over R shards answers exactly what one GPU answers (Def. 1): the library
routes each query to the owner of its cell, the owner's bounded requests go to the shards its
search entered, replies are merged (first-k of the union) and the answers return to their
origin rows.  With one GPU available the same protocol runs
  * in one process over R shards on cuda:0 (opts.n_gpus = R, devices = [0]*R: the loopback
    exchange -- peer copies between the shards' buffers), and
  * in R processes sharing cuda:0, each rank's handle built with opts.n_ranks / rank and a
    torch.distributed (gloo) all-to-all as opts.exchange (the multi-process path; NCCL is
    the same code with ncclSend / ncclRecv as the transport).
The NCCL transport itself needs distinct GPUs: covered when the box has >= 2.
"""
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


def _same(got, ref, what):
    go, gd = got
    ro, rd = ref
    bad = np.flatnonzero(~((go == ro).all(1) & (gd == rd).all(1)))
    assert len(bad) == 0, (f"{what}: {len(bad)} rows differ; first {bad[0]}: got {list(zip(gd[bad[0]], go[bad[0]]))} "
                           f"ref {list(zip(rd[bad[0]], ro[bad[0]]))}")


@pytest.mark.parametrize("n", [1, 2, 4, 8])
def test_loopback_index_bit_exact(gg, n):
    """R = 1, 2, 4, 8 shards in one process on one GPU: every row the oracle's; the R = 1
    handle is the plain single-GPU index."""
    g = synth.table_ii_graph("NY", scale=0.2)
    walk = synth.RandomWalk(g, 20_000, inject=True)
    opts = dict(max_objects=20_000)
    if n > 1:
        opts.update(n_gpus=n, devices=[0] * n)
    grid = gg.GGrid(g, 256, **opts)
    hist = []
    for it in range(3):
        u = walk.ticks(3)
        hist.append(u)
        grid.ingest(u)
        q = synth.queries(g, 700, seed=40 + it)
        _same(grid.knn(q, 10), oracle.knn_from_updates(g, np.concatenate(hist), q, 10), f"R={n} round {it}")
    st = grid.stats()
    assert st["n_shards"] == n
    if n > 1:
        assert st["exchange_kind"] == gg.GGRID_EXCHANGE_LOOPBACK
        assert st["objects_written"] > 0
    grid.close()


@pytest.mark.parametrize("mode", [1, 2, 3, 4])
def test_loopback_ingest_paths(gg, mode):
    """Every ingest path in sharded mode (4 shards): updates of other shards' cells only raise the
    replicated object table (and mark the cell an object leaves STALE on its owner) -- the cell-hash
    launch (1), the direct launch (2), the three launches (3) and the sort-by-cell path (4) all give
    the oracle's answers."""
    g = synth.table_ii_graph("NY", scale=0.2)
    walk = synth.RandomWalk(g, 20_000, inject=True)
    grid = gg.GGrid(g, 256, max_objects=20_000, n_gpus=4, devices=[0] * 4, ingest_kernels=mode)
    hist = []
    for it in range(3):
        u = walk.ticks(2 + it)
        hist.append(u)
        grid.ingest(u)
        q = synth.queries(g, 500, seed=70 + it)
        _same(grid.knn(q, 9), oracle.knn_from_updates(g, np.concatenate(hist), q, 9), f"mode {mode} round {it}")
    grid.close()


def test_loopback_edge_cases(gg):
    """Fewer queries than shards (empty origin shares), k beyond the objects (padding), ties
    (lattice weights 1..4), device inputs and outputs, a flush_all and the per-cell dump routed
    to the owner shard."""
    import torch

    g = synth.lattice_graph(32, 32, 1, 4)
    upd = synth.RandomWalk(g, 100, inject=True).ticks(10)
    grid = gg.GGrid(g, 16, max_objects=128, n_gpus=4, devices=[0, 0, 0, 0])
    grid.ingest(torch.from_numpy(upd.view(np.int32)).cuda())
    q = synth.queries(g, 3)
    _same(grid.knn(q, 3), oracle.knn_from_updates(g, upd, q, 3), "3 queries over 4 shards")
    q = synth.queries(g, 100, seed=9)
    _same(grid.knn(q, 130), oracle.knn_from_updates(g, upd, q, 130), "k > objects")
    qd = torch.from_numpy(q.view(np.int32)).cuda()
    oo = torch.empty((100, 5), dtype=torch.int32, device="cuda")
    od = torch.empty_like(oo)
    grid.knn(qd, 5, oo, od)
    _same((oo.cpu().numpy().view(np.uint32), od.cpu().numpy().view(np.uint32)),
          oracle.knn_from_updates(g, upd, q, 5), "device buffers")
    grid.flush_all()
    ids, e, d = oracle.snapshot_objects(upd)
    vcell = grid.vertex_cell()
    rows = []
    for c in range(grid.stats()["n_cells"]):
        o, e_, d_ = grid.cell_objects(c)
        assert np.all(vcell[g["src"][e_]] == c)
        rows += list(zip(o.tolist(), e_.tolist(), d_.tolist()))
    assert sorted(rows) == sorted(zip(ids.tolist(), e.tolist(), d.tolist()))
    with pytest.raises(gg.GGridError):
        grid.knn_ex(q, 3)  # single-shard primitives are refused on a multi-GPU handle
    grid.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_worker(rank, world, port, q_out):
    import torch
    import torch.distributed as dist

    import paper_conf_icde_li0qhdy18_b200 as gg

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        _rank_body(rank, world, q_out)
    except Exception as e:  # (reported, so the test fails instead of waiting for a result)
        q_out.put((rank, -1, repr(e), 0))
        raise
    finally:
        dist.destroy_process_group()


def _rank_body(rank, world, q_out):
    import torch

    import paper_conf_icde_li0qhdy18_b200 as gg

    torch.cuda.set_device(0)
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 3000, inject=True)
    grid = gg.GGrid(g, 128, max_objects=3000, n_ranks=world, rank=rank, exchange=gg.alltoall_callback())
    hist = []
    bad_total = 0
    for it in range(2):
        u = walk.ticks(2)
        hist.append(u)
        grid.ingest(u)  # every rank ingests the whole stream
        nq = 150 + 37 * rank  # different batch sizes per rank
        q = synth.queries(g, nq, seed=1000 * rank + it)
        go, gd = grid.knn(q, 8)  # collective
        ro, rd = oracle.knn_from_updates(g, np.concatenate(hist), q, 8)
        bad_total += int((~((go == ro).all(1) & (gd == rd).all(1))).sum())
    st = grid.stats()
    q_out.put((rank, bad_total, int(st["n_shards"]), int(st["exchange_kind"])))
    grid.close()


@pytest.mark.parametrize("world", [2, 3])
def test_multiprocess_ranks_callback_exchange(gg, world):
    """One process per rank (sharing cuda:0), opts.n_ranks / rank with a gloo all-to-all as the
    exchange: each rank's own batch answered exactly, per-rank batch sizes differ."""
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q_out = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_worker, args=(r, world, port, q_out)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q_out.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
    assert all(bad == 0 for _, bad, _, _ in res), res
    assert all(ns == world and kind == 3 for _, _, ns, kind in res), res


def test_nccl_unique_id(gg):
    try:
        uid = gg.ggrid_nccl_unique_id()
    except gg.GGridError as e:
        assert e.rc == gg.GGRID_ENCCL
        pytest.skip("libnccl not loadable")
    assert len(uid) == 128 and any(uid)


def test_nccl_in_process_distinct_gpus(gg):
    """NCCL transport (ncclCommInitAll over distinct devices): needs >= 2 GPUs."""
    import torch

    n = torch.cuda.device_count()
    if n < 2:
        pytest.skip("one GPU: the NCCL transport needs distinct devices (loopback covers the protocol)")
    g = synth.table_ii_graph("NY", scale=0.2)
    upd = synth.RandomWalk(g, 20_000).ticks(4)
    grid = gg.GGrid(g, 256, max_objects=20_000, n_gpus=n, exchange_kind=gg.GGRID_EXCHANGE_NCCL)
    grid.ingest(upd)
    q = synth.queries(g, 500)
    _same(grid.knn(q, 10), oracle.knn_from_updates(g, upd, q, 10), f"NCCL x{n}")
    assert grid.stats()["exchange_kind"] == gg.GGRID_EXCHANGE_NCCL
    grid.close()
