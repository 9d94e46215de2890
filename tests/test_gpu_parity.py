"""Parity of the CUDA path (through the C ABI) against the CPU oracle (-m gpu).

The bar (north_star): integer work, so bit-exact — identical object ids AND
distances per query, ties broken by id, padding identical.
"""
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


def _oracle(g, upd, q, k, mode=oracle.FULL):
    return oracle.knn_from_updates(g, upd, q, k, mode=mode)


def _assert_same(got, ref, msg=""):
    go, gd = got
    ro, rd = ref
    if not (np.array_equal(go, ro) and np.array_equal(gd, rd)):
        bad = np.flatnonzero(~((go == ro).all(1) & (gd == rd).all(1)))
        i = int(bad[0])
        raise AssertionError(f"{msg}: {len(bad)} rows differ; first row {i}: got {list(zip(gd[i], go[i]))} "
                             f"ref {list(zip(rd[i], ro[i]))}")


# ---------------------------------------------------------------------------------- C0
@pytest.mark.parametrize("cell_size", [1, 16, 64, 1024])
def test_c0_knn_bit_exact(gg, cell_size):
    """BASELINE configs[0]: 32x32 lattice, w in {1..4} (ties), 100 objects, 1k cached updates
    with late / duplicate timestamps, 100 queries; every cell_size gives the oracle's answer
    (partition independence)."""
    g = synth.lattice_graph(32, 32, 1, 4)
    upd = synth.RandomWalk(g, 100, inject=True).ticks(10)
    q = synth.queries(g, 100)
    grid = gg.GGrid(g, cell_size, max_objects=128)
    grid.ingest(upd)
    for k in (1, 3, 10, 100, 130):
        _assert_same(grid.knn(q, k), _oracle(g, upd, q, k), f"cs={cell_size} k={k}")
    grid.close()


def test_c0_interleaved_rounds_lazy_equals_eager(gg):
    """Interleaved ingest / query rounds; a lazy handle and an eager one (flush_all after
    every ingest) agree with the oracle's snapshot at every round."""
    g = synth.lattice_graph(32, 32, 1, 4)
    walk = synth.RandomWalk(g, 100, inject=True)
    lazy = gg.GGrid(g, 16, max_objects=128)
    eager = gg.GGrid(g, 16, max_objects=128)
    hist = []
    for r in range(8):
        u = walk.ticks(3)
        hist.append(u)
        lazy.ingest(u)
        eager.ingest(u)
        eager.flush_all()
        allu = np.concatenate(hist)
        q = synth.queries(g, 64, seed=100 + r)
        ref = _oracle(g, allu, q, 5)
        _assert_same(lazy.knn(q, 5), ref, f"lazy round {r}")
        _assert_same(eager.knn(q, 5), ref, f"eager round {r}")
    lazy.close()
    eager.close()


@pytest.mark.parametrize("kernel", ["auto", "ring", "streaming", "warp"])
def test_flush_parity_and_cells(gg, kernel, monkeypatch):
    """After ggrid_flush_all the cells' object lists are exactly the oracle's latest-per-object
    snapshot, each object once, in the cell of its arc's source vertex; flushing twice is a
    no-op (idempotent).  Every flush kernel (the bulk-copy ring, the streaming one and the
    warp-per-cell one; GGRID_FLUSH_KERNEL forces one, `auto` picks by log length per cell)."""
    monkeypatch.setenv("GGRID_FLUSH_KERNEL", {"auto": "0", "ring": "1", "streaming": "2", "warp": "3"}[kernel])
    g = synth.table_ii_graph("NY", scale=0.05)
    upd = synth.RandomWalk(g, 2000, inject=True).ticks(12)
    grid = gg.GGrid(g, 256, max_objects=4096)
    for part in np.array_split(upd, 5):
        grid.ingest(part)
    grid.flush_all()
    vcell = grid.vertex_cell()
    n_cells = grid.stats()["n_cells"]

    def dump():
        rows = []
        for c in range(n_cells):
            o, e, d = grid.cell_objects(c)
            assert np.all(vcell[g["src"][e]] == c)
            rows += list(zip(o.tolist(), e.tolist(), d.tolist()))
        return sorted(rows)

    got = dump()
    ids, e, d = oracle.snapshot_objects(upd)
    assert got == sorted(zip(ids.tolist(), e.tolist(), d.tolist()))
    grid.flush_all()
    assert dump() == got
    grid.close()


def test_batch_independence_and_pointer_kinds(gg):
    import torch

    g = synth.table_ii_graph("NY", scale=0.05)
    upd = synth.RandomWalk(g, 1000).ticks(5)
    q = synth.queries(g, 200)
    k = 7
    ref = _oracle(g, upd, q, k)
    grid = gg.GGrid(g, 256, max_objects=1024)
    grid.ingest(torch.from_numpy(upd.view(np.int32)).cuda())  # device input
    one = [grid.knn(q[i:i + 1], k) for i in range(0, 40)]
    _assert_same((np.concatenate([a for a, _ in one]), np.concatenate([b for _, b in one])),
                 (ref[0][:40], ref[1][:40]), "Q=1 calls")
    qo = torch.empty((len(q), k), dtype=torch.int32, device="cuda")
    qd = torch.empty((len(q), k), dtype=torch.int32, device="cuda")
    grid.knn(torch.from_numpy(q.view(np.int32)).cuda(), k, qo, qd)  # device in / out
    _assert_same((qo.cpu().numpy().view(np.uint32), qd.cpu().numpy().view(np.uint32)), ref, "device io")
    po = torch.empty((len(q), k), dtype=torch.int32).pin_memory()
    pd = torch.empty((len(q), k), dtype=torch.int32).pin_memory()
    grid.knn(torch.from_numpy(q.view(np.int32)).pin_memory(), k, po, pd)  # pinned host
    _assert_same((po.numpy().view(np.uint32), pd.numpy().view(np.uint32)), ref, "pinned io")
    grid.close()


# ----------------------------------------------------------------- tiny graphs / edge cases
@pytest.mark.parametrize("seed", range(40))
def test_random_digraphs(gg, seed):
    """Random directed multigraphs with self-loops, unreachable parts and ties."""
    rng = np.random.default_rng(500 + seed)
    V = int(rng.integers(2, 40))
    A = int(rng.integers(1, 4 * V))
    g = dict(n_vertices=V, src=rng.integers(0, V, A).astype(np.uint32),
             dst=rng.integers(0, V, A).astype(np.uint32), w=rng.integers(1, 6, A).astype(np.uint32))
    n_obj = int(rng.integers(1, 30))
    n_upd = int(rng.integers(1, 200))
    upd = np.zeros((n_upd, 4), np.uint32)
    upd[:, 0] = rng.integers(0, n_obj, n_upd)
    upd[:, 1] = rng.integers(0, A, n_upd)
    upd[:, 2] = (rng.random(n_upd) * g["w"][upd[:, 1]]).astype(np.uint32)
    upd[:, 3] = rng.integers(0, 20, n_upd)
    q = np.zeros((30, 2), np.uint32)
    q[:, 0] = rng.integers(0, A, 30)
    q[:, 1] = (rng.random(30) * g["w"][q[:, 0]]).astype(np.uint32)
    for cs in (1, 3, V):
        grid = gg.GGrid(g, cs, max_objects=64, delta=int(rng.integers(1, 8)))
        for part in np.array_split(upd, 3):
            if len(part):
                grid.ingest(part)
        for k in (1, 4, 40):
            _assert_same(grid.knn(q, k), _oracle(g, upd, q, k), f"seed={seed} cs={cs} k={k}")
        grid.close()


def test_fig1_fixture_through_library(gg):
    d, g = synth.fig1_fixture()
    W = d["lattice"]["width"]

    def arc(a, b):
        return int(np.flatnonzero((g["src"] == a[1] * W + a[0]) & (g["dst"] == b[1] * W + b[0]))[0])

    upd = np.array([[o["id"], arc(o["from"], o["to"]), o["offset"], 0] for o in d["objects"]], np.uint32)
    q = np.array([[arc(d["query"]["from"], d["query"]["to"]), d["query"]["offset"]]], np.uint32)
    grid = gg.GGrid(g, 8, max_objects=16)
    grid.ingest(upd)
    o, _ = grid.knn(q, 3)
    assert o[0].tolist() == d["paper_answer"]  # <o5, o2, o4>
    o, dist = grid.knn(q, 9)
    assert [[int(a), int(b)] for a, b in zip(o[0], dist[0])] == d["hand_order"]
    grid.close()


def test_u32_distance_range(gg):
    big = 1 << 31
    g = dict(n_vertices=3, src=np.array([0, 1], np.uint32), dst=np.array([1, 2], np.uint32),
             w=np.array([big, big], np.uint32))
    upd = np.array([[1, 1, big - 2, 0], [2, 1, big - 1, 0], [3, 0, 5, 0]], np.uint32)
    grid = gg.GGrid(g, 2, max_objects=8)
    grid.ingest(upd)
    o, d = grid.knn(np.array([[0, 0]], np.uint32), 3)
    assert o.tolist() == [[3, 1, gg.PAD]] and d.tolist() == [[5, (1 << 32) - 2, gg.PAD]]
    grid.close()


def test_delta_independence(gg):
    g = synth.table_ii_graph("NY", scale=0.03)
    upd = synth.RandomWalk(g, 500, inject=True).ticks(4)
    q = synth.queries(g, 100)
    ref = _oracle(g, upd, q, 10)
    for delta in (1, 97, 1000, 1 << 30):
        grid = gg.GGrid(g, 128, max_objects=512, delta=delta)
        grid.ingest(upd)
        _assert_same(grid.knn(q, 10), ref, f"delta={delta}")
        grid.close()


def test_large_k_and_sparse_objects_use_every_level(gg):
    """k above the level-0 limit and fewer reachable objects than k: levels 1 and 2."""
    g = synth.table_ii_graph("NY", scale=0.05)
    upd = synth.RandomWalk(g, 40).ticks(2)
    q = synth.queries(g, 20)
    grid = gg.GGrid(g, 512, max_objects=64, max_k=1024)
    grid.ingest(upd)
    for k in (129, 600):
        _assert_same(grid.knn(q, k), _oracle(g, upd, q, k), f"k={k}")
    st = grid.stats()
    assert st["kernel_launches"]["expand_big"] > 0
    grid.close()


def test_einval_rejects_batch_atomically(gg):
    g = synth.lattice_graph(8, 8, 1, 4)
    grid = gg.GGrid(g, 16, max_objects=32, max_k=8)
    good = synth.RandomWalk(g, 20).ticks(2)
    grid.ingest(good)
    for bad_row in ([40, 0, 0, 0], [1, len(g["src"]), 0, 0], [1, 3, int(g["w"][3]), 0]):
        bad = np.concatenate([good[:5], np.array([bad_row], np.uint32), good[5:9]])
        with pytest.raises(gg.GGridError) as e:
            grid.ingest(bad)
        assert e.value.rc == gg.GGRID_EINVAL
    q = synth.queries(g, 10)
    _assert_same(grid.knn(q, 4), _oracle(g, good, q, 4), "after rejected batches")
    for k in (0, 9):
        with pytest.raises(gg.GGridError):
            grid.knn(q, k)
    with pytest.raises(gg.GGridError):
        grid.knn(np.array([[len(g["src"]), 0]], np.uint32), 2)
    with pytest.raises(gg.GGridError):
        grid.knn(np.array([[3, int(g["w"][3])]], np.uint32), 2)
    assert grid.stats()["n_updates"] == len(good)
    grid.close()


def test_garbage_collection_keeps_answers(gg):
    g = synth.table_ii_graph("NY", scale=0.03)
    walk = synth.RandomWalk(g, 800, inject=True)
    grid = gg.GGrid(g, 128, max_objects=1024, log_capacity=12_000)
    hist = []
    for r in range(12):
        u = walk.ticks(3)
        hist.append(u)
        grid.ingest(u)
        q = synth.queries(g, 50, seed=7 + r)
        _assert_same(grid.knn(q, 6), _oracle(g, np.concatenate(hist), q, 6), f"round {r}")
    assert grid.stats()["gc_runs"] > 0
    grid.close()


def test_async_ingest_deferred_errors(gg):
    """opts.async_ingest: ggrid_ingest returns without a host round trip; a bad batch is still
    rejected whole on the device and its EINVAL surfaces once, at the next ggrid_sync (or the
    next ggrid_ingest); answers are the oracle's on the accepted batches."""
    g = synth.lattice_graph(8, 8, 1, 4)
    grid = gg.GGrid(g, 16, max_objects=32, max_k=8, async_ingest=True)
    walk = synth.RandomWalk(g, 20, inject=True)
    good = [walk.ticks(2)]
    grid.ingest(good[0])
    bad = np.concatenate([good[0][:5], np.array([[1, len(g["src"]), 0, 0]], np.uint32)])
    grid.ingest(bad)  # accepted for now: validated on the device
    q = synth.queries(g, 10)
    _assert_same(grid.knn(q, 4), _oracle(g, good[0], q, 4), "rejected batch not visible")
    with pytest.raises(gg.GGridError) as e:
        grid.sync()
    assert e.value.rc == gg.GGRID_EINVAL
    grid.sync()  # reported once
    # the next ingest reports a deferred error instead of the sync
    grid.ingest(np.array([[40, 0, 0, 0]], np.uint32))
    grid.knn(q, 4)  # (syncs: the mirror now holds the rejection)
    with pytest.raises(gg.GGridError) as e:
        grid.ingest(walk.ticks(1))
    assert e.value.rc == gg.GGRID_EINVAL
    good.append(walk.ticks(2))
    grid.ingest(good[-1])
    grid.sync()
    _assert_same(grid.knn(q, 4), _oracle(g, np.concatenate(good), q, 4), "after deferred errors")
    grid.close()


def test_async_ingest_streams_and_gc(gg):
    """Asynchronous ingest across many batches with no sync in between, under arena pressure
    (garbage collection must see the pending batches' records): bit-exact at every query."""
    g = synth.table_ii_graph("NY", scale=0.03)
    walk = synth.RandomWalk(g, 800, inject=True)
    grid = gg.GGrid(g, 128, max_objects=1024, log_capacity=12_000, async_ingest=True)
    hist = []
    for r in range(10):
        for _ in range(3):  # several batches queued back to back
            u = walk.ticks(1)
            hist.append(u)
            grid.ingest(u)
        q = synth.queries(g, 50, seed=70 + r)
        _assert_same(grid.knn(q, 6), _oracle(g, np.concatenate(hist), q, 6), f"round {r}")
    grid.sync()
    assert grid.stats()["gc_runs"] > 0
    grid.close()


# ----------------------------------------------------------------- BASELINE-scale configs
def test_c1_ny_bit_exact(gg):
    """configs[1] at full size: NY-shaped graph, 10k objects, 1M cached updates, k=10;
    every one of 2,000 queries checked against the full-Dijkstra oracle."""
    g = synth.config_graph("C1")
    upd = synth.RandomWalk(g, 10_000, inject=True).ticks(100)
    q = synth.queries(g, 2000)
    grid = gg.GGrid(g, 1024, max_objects=10_000)
    grid.ingest(upd)
    got = grid.knn(q, 10)
    _assert_same(got, _oracle(g, upd, q, 10), "C1")
    grid.close()


def test_c2_fla_k_sweep(gg):
    """configs[2]: FLA-shaped, 100k objects, k = 10..50 (sampled 300 queries, EARLY oracle
    cross-checked against FULL on a subset in test_oracle)."""
    g = synth.config_graph("C2")
    upd = synth.RandomWalk(g, 100_000).ticks(10)
    q = synth.queries(g, 300)
    grid = gg.GGrid(g, 1024, max_objects=100_000)
    grid.ingest(upd)
    for k in (10, 20, 30, 40, 50):
        _assert_same(grid.knn(q, k), _oracle(g, upd, q, k, mode=oracle.EARLY), f"C2 k={k}")
    grid.close()


# ------------------------------------------------------------ flush paths and bench config
def test_flush_histogram_and_global_counter_paths(gg):
    """cell_size > 4096 (per-vertex counters in global memory) and > 128 winners per cell
    (counter + scan indexing instead of ranks)."""
    g = synth.table_ii_graph("NY", scale=0.03)
    upd = synth.RandomWalk(g, 3000, inject=True).ticks(6)
    q = synth.queries(g, 200)
    for cs in (5000, 2048):
        grid = gg.GGrid(g, cs, max_objects=4096)
        grid.ingest(upd)
        _assert_same(grid.knn(q, 8), _oracle(g, upd, q, 8), f"cs={cs}")
        grid.close()


def test_flush_long_chains_and_overflow(gg):
    """40 ingest batches without a query (chains longer than the 32-extent gather), and one
    cell holding far more objects than the flush's winner staging (re-stream fallback)."""
    g = synth.table_ii_graph("NY", scale=0.03)
    grid = gg.GGrid(g, 64, max_objects=8192)
    vcell = grid.vertex_cell()
    # crowd 1500 objects onto the arcs leaving cell 0's vertices
    hot = np.flatnonzero(vcell[g["src"]] == 0)
    rng = np.random.default_rng(9)
    n_hot = 1500
    e = hot[rng.integers(0, len(hot), n_hot)].astype(np.uint32)
    d = (rng.random(n_hot) * g["w"][e]).astype(np.uint32)
    crowd = np.stack([np.arange(n_hot, dtype=np.uint32), e, d, np.zeros(n_hot, np.uint32)], 1)
    walk = synth.RandomWalk(g, 600, obj_ids=np.arange(n_hot, n_hot + 600, dtype=np.uint32))
    hist = [crowd]
    grid.ingest(crowd)
    for _ in range(40):
        u = walk.tick()
        hist.append(u)
        grid.ingest(u)
    allu = np.concatenate(hist)
    q = synth.queries(g, 150)
    q[:20, 0] = hot[:20]  # queries right at the crowded cell
    q[:20, 1] = 0
    _assert_same(grid.knn(q, 12), _oracle(g, allu, q, 12), "long chains + crowded cell")
    grid.close()


def test_flush_spill_paths(gg):
    """Many objects per cell (the wider staging variant): one cell with more winners than the
    shared-memory staging (positions spill to global memory), one beyond the spill area too
    (re-stream), plus a random walk; GC (full v_obj rewrite) over the same state."""
    g = synth.table_ii_graph("NY", scale=0.03)
    grid = gg.GGrid(g, 64, max_objects=30_000, log_capacity=120_000)  # small: forces GC
    vcell = grid.vertex_cell()
    rng = np.random.default_rng(11)
    parts, oid = [], 0
    for cell, n_hot in ((0, 900), (1, 3000)):
        hot = np.flatnonzero(vcell[g["src"]] == cell)
        e = hot[rng.integers(0, len(hot), n_hot)].astype(np.uint32)
        d = (rng.random(n_hot) * g["w"][e]).astype(np.uint32)
        parts.append(np.stack([np.arange(oid, oid + n_hot, dtype=np.uint32), e, d,
                               np.full(n_hot, 5, np.uint32)], 1))
        oid += n_hot
    walk = synth.RandomWalk(g, 18_000, obj_ids=np.arange(oid, oid + 18_000, dtype=np.uint32))
    hist = parts + [walk.ticks(3)]
    for u in hist:
        grid.ingest(u)
    q = synth.queries(g, 200)
    for i, cell in enumerate((0, 1)):
        hot = np.flatnonzero(vcell[g["src"]] == cell)
        q[20 * i:20 * i + 20, 0] = hot[:20]
        q[20 * i:20 * i + 20, 1] = 0
    allu = np.concatenate(hist)
    _assert_same(grid.knn(q, 40), _oracle(g, allu, q, 40), "spill + re-stream")
    u = walk.ticks(2)
    allu = np.concatenate([allu, u])
    grid.ingest(u)
    grid.flush_all()
    _assert_same(grid.knn(q, 40), _oracle(g, allu, q, 40), "after flush_all")
    st = grid.stats()
    assert st["kernel_launches"]["flush"] >= 2 and st["gc_runs"] >= 1, st
    grid.close()


def test_expiry_honoured_is_exact(gg):
    """t_delta expiry (P@20631-21157, reading R21) when every object reports within t_delta:
    extents older than t_now - t_delta are dropped unread and the answers stay exact."""
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 3000)  # every object reports once per tick (t = tick*1000+U[0,999])
    grid = gg.GGrid(g, 256, max_objects=3000, t_delta=2000)
    hist = []
    for tick in range(12):
        u = walk.tick()
        hist.append(u)
        grid.ingest(u)
        if tick == 5:  # clean some cells midway
            grid.knn(synth.queries(g, 20, seed=5), 5)
    q = synth.queries(g, 300)
    allu = np.concatenate(hist)
    _assert_same(grid.knn(q, 16), _oracle(g, allu, q, 16), "expiry, honoured")
    st = grid.stats()
    assert st["t_now"] == int(allu[:, 3].max()) and st["t_delta"] == 2000
    assert st["records_expired"] > 0, st
    grid.flush_all()
    _assert_same(grid.knn(q, 16), _oracle(g, allu, q, 16), "expiry, after flush_all")
    grid.close()


def test_expiry_drops_silent_objects(gg):
    """An object silent for longer than t_delta (the paper's reporting assumption violated,
    P@20935) disappears when its cached extent expires; without expiry it stays."""
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 800, obj_ids=np.arange(1, 801, dtype=np.uint32))
    e0 = np.uint32(17)
    silent = np.array([[0, e0, 0, 0]], np.uint32)  # object 0 at t = 0, alone in its batch
    ticks = []
    for _ in range(6):
        u = walk.tick()
        u[:, 3] += 1000  # the walk starts at t = 1000
        ticks.append(u)
    q = np.array([[e0, 0]], np.uint32)  # right at object 0
    for t_delta, expect_silent in ((0, True), (2000, False)):
        grid = gg.GGrid(g, 256, max_objects=801, t_delta=t_delta)
        for u in [silent] + ticks:
            grid.ingest(u)
        go, gd = grid.knn(q, 5)
        ref_upd = np.concatenate(([silent] if expect_silent else []) + ticks)
        _assert_same((go, gd), _oracle(g, ref_upd, q, 5), f"t_delta={t_delta}")
        assert (0 in go[0]) == expect_silent
        grid.close()


def test_bench_configuration_steady_state(gg):
    """The launch configuration bench.py times (C1: NY graph, cell_size 1024, profile mode on a
    caller stream, 1M updates + 10k queries per step): every query of the first step and 1,000
    sampled queries of two further steps, bit-exact."""
    import torch

    g = synth.config_graph("C1")
    walk = synth.RandomWalk(g, 10_000)
    stream = torch.cuda.Stream()
    grid = gg.GGrid(g, 1024, max_objects=10_000, profile=True, stream=stream.cuda_stream)
    out_o = torch.empty((10_000, 10), dtype=torch.int32, device="cuda")
    out_d = torch.empty((10_000, 10), dtype=torch.int32, device="cuda")
    hist = []
    for step in range(3):
        u = walk.ticks(100)
        hist.append(u)
        q = synth.queries(g, 10_000, seed=synth.SEED_QUERIES + step)
        grid.ingest(torch.from_numpy(u.view(np.int32)).cuda())
        grid.knn(torch.from_numpy(q.view(np.int32)).cuda(), 10, out_o, out_d)
        torch.cuda.synchronize()
        go = out_o.cpu().numpy().view(np.uint32)
        gd = out_d.cpu().numpy().view(np.uint32)
        sel = np.arange(10_000) if step == 0 else np.random.default_rng(step).choice(10_000, 1000, replace=False)
        ro, rd = _oracle(g, np.concatenate(hist), q[sel], 10)
        _assert_same((go[sel], gd[sel]), (ro, rd), f"step {step}")
    grid.close()


def test_usa_shaped_sampled(gg):
    """configs[3] shape at 1/10 scale (2.4M vertices, 5.8M arcs): 100k objects, 64 cached
    updates each, 65,536 queries; 200 sampled rows against the oracle (EARLY) and 10 (FULL)."""
    g = synth.table_ii_graph("USA", scale=0.1)
    upd = synth.RandomWalk(g, 100_000).ticks(64)
    grid = gg.GGrid(g, 1024, max_objects=100_000, log_capacity=8_000_000)
    grid.ingest(upd)
    q = synth.queries(g, 65536)
    go, gd = grid.knn(q, 10)
    sel = np.linspace(0, 65535, 200).astype(np.int64)
    _assert_same((go[sel], gd[sel]), _oracle(g, upd, q[sel], 10, mode=oracle.EARLY), "USA/10 early")
    _assert_same((go[sel[:10]], gd[sel[:10]]), _oracle(g, upd, q[sel[:10]], 10), "USA/10 full")
    grid.close()


def test_pipelined_ingest_stage_commit(gg):
    """ggrid_ingest_stage/commit (P@45017-45625 pipelined transfer): a knn issued between
    stage and commit answers on the snapshot without the staged batch; after the commit it
    includes it; the stage/commit misuse errors."""
    import torch

    g = synth.table_ii_graph("NY", scale=0.03)
    walk = synth.RandomWalk(g, 500, inject=True)
    u1, u2, u3 = walk.ticks(3), walk.ticks(3), walk.ticks(3)
    q = synth.queries(g, 100)
    grid = gg.GGrid(g, 128, max_objects=512)
    with pytest.raises(gg.GGridError):
        grid.ingest_commit()  # nothing staged
    grid.ingest(u1)
    grid.ingest_stage(torch.from_numpy(u2.view(np.int32)).pin_memory())
    grid.ingest_stage(u3)  # pageable host memory also works
    with pytest.raises(gg.GGridError):
        grid.ingest_stage(u3)  # both buffers staged
    _assert_same(grid.knn(q, 6), _oracle(g, u1, q, 6), "before commit")
    grid.ingest_commit()
    _assert_same(grid.knn(q, 6), _oracle(g, np.concatenate([u1, u2]), q, 6), "after commit 1")
    grid.ingest_commit()
    _assert_same(grid.knn(q, 6), _oracle(g, np.concatenate([u1, u2, u3]), q, 6), "after commit 2")
    assert grid.stats()["n_updates"] == len(u1) + len(u2) + len(u3)
    grid.close()


def test_pipelined_queries_stage_commit(gg):
    """ggrid_query_stage / ggrid_knn_commit (two-deep query staging on the copy stream),
    interleaved with staged update batches: every committed batch answers the snapshot of the
    updates committed before it, bit-exact."""
    import torch

    g = synth.table_ii_graph("NY", scale=0.03)
    walk = synth.RandomWalk(g, 500, inject=True)
    grid = gg.GGrid(g, 128, max_objects=512, async_ingest=True)
    ups = [walk.ticks(2) for _ in range(5)]
    qs = [synth.queries(g, 40 + 7 * i, seed=300 + i) for i in range(5)]
    hu = [torch.from_numpy(u.view(np.int32)).pin_memory() for u in ups]
    hq = [torch.from_numpy(q.view(np.int32)).pin_memory() for q in qs]
    k = 5
    grid.ingest_stage(hu[0])
    grid.query_stage(hq[0])
    for s in range(5):
        grid.ingest_commit()
        if s + 1 < 5:
            grid.ingest_stage(hu[s + 1])
            grid.query_stage(hq[s + 1])
        o = torch.empty((len(qs[s]), k), dtype=torch.int32).pin_memory()
        d = torch.empty((len(qs[s]), k), dtype=torch.int32).pin_memory()
        grid.knn_commit(k, o, d)
        ref = _oracle(g, np.concatenate(ups[: s + 1]), qs[s], k)
        _assert_same((o.numpy().view(np.uint32), d.numpy().view(np.uint32)), ref, f"batch {s}")
    with pytest.raises(gg.GGridError):
        grid.knn_commit(k, o, d)  # nothing staged
    grid.close()


def test_ladder_boundaries_and_promotions(gg):
    """k at the capacity-ladder boundaries (32 | 33: level 0 | level 1's 128 candidates; 96 | 97:
    level 1 | level 2) and a density where the starting level is the 4-warp CTA variant
    (expected ball ~440 vertices) but the sparsest queries overflow its 1,024-slot table and are
    promoted to the level running beside it: every row the oracle's."""
    g = synth.table_ii_graph("NY", scale=0.2)
    upd = synth.RandomWalk(g, 1200, inject=True).ticks(3)
    q = synth.queries(g, 600)
    grid = gg.GGrid(g, 256, max_objects=2048)
    grid.ingest(upd)
    _assert_same(grid.knn(q, 10), _oracle(g, upd, q, 10), "k=10")
    promoted = grid.stats()["expand_promotions"]
    for k in (32, 33, 96, 97):
        _assert_same(grid.knn(q[:200], k), _oracle(g, upd, q[:200], k), f"k={k}")
    assert promoted > 0  # (3 with these seeds: the promotion path ran)
    grid.close()


def test_resumed_promotions_one_warp_level(gg):
    """The one-warp starting level (dense objects: expected ball ~90 vertices) with every object in
    the western half of the graph: eastern queries overflow the 704-slot table mid-search and are
    promoted WITH their state (knn.cu promote_export) to the chained level, which re-hashes it and
    continues; those that overflow there too restart at the levels above.  Every row the
    oracle's, and the resume path ran."""
    g = synth.table_ii_graph("NY", scale=0.2)
    rng = np.random.default_rng(11)
    west = np.nonzero(g["x"][g["src"]] < np.quantile(g["x"], 0.5))[0]
    n = 6000
    arc = rng.choice(west, n).astype(np.int64)
    off = np.minimum((rng.random(n) * g["w"][arc]).astype(np.int64), g["w"][arc].astype(np.int64) - 1)
    upd = np.stack([np.arange(n), arc, off, np.ones(n, np.int64)], 1).astype(np.uint32)
    q = synth.queries(g, 1500, seed=77)
    grid = gg.GGrid(g, 256, max_objects=n)
    grid.ingest(upd)
    for k in (10, 20):
        _assert_same(grid.knn(q, k), _oracle(g, upd, q, k), f"k={k}")
    st = grid.stats()
    assert st["expand_promotions"] > 0
    assert st["expand_resumes"] > 0
    grid.close()


def test_moved_objects_leave_clean_cells_stale(gg):
    """Objects jumping between cells every round (uniform random relocation, 4-vertex cells):
    the cell an object left is marked STALE at ingest and re-cleaned before its list is read,
    so answers stay exact without the per-object validity gather (reading R8).  Queries are
    interleaved with the jumps; some rounds re-send older timestamps (late arrivals)."""
    g = synth.table_ii_graph("NY", scale=0.01)
    rng = np.random.default_rng(5)
    n_obj = 300
    grid = gg.GGrid(g, 4, max_objects=n_obj)
    hist = []
    for r in range(12):
        arc, off = synth.random_locations(g, n_obj, rng)
        t = np.full(n_obj, 1000 * r, np.uint32) if r % 4 != 3 else np.full(n_obj, 1000 * (r - 2), np.uint32)
        u = np.stack([np.arange(n_obj, dtype=np.uint32)[rng.permutation(n_obj)], arc, off, t], 1).astype(np.uint32)
        u[:, 1] = arc[u[:, 0]]
        u[:, 2] = off[u[:, 0]]
        hist.append(u)
        grid.ingest(u)
        q = synth.queries(g, 150, seed=600 + r)
        _assert_same(grid.knn(q, 7), _oracle(g, np.concatenate(hist), q, 7), f"round {r}")
    grid.close()


@pytest.mark.parametrize("kernel", ["1", "2", "3"])
def test_flush_kernels_interleaved_rounds(gg, kernel, monkeypatch):
    """Interleaved ingest / query rounds with either flush kernel forced (long chains of small
    extents, STALE cells, cleaned lists re-read): every round the oracle's answer."""
    monkeypatch.setenv("GGRID_FLUSH_KERNEL", kernel)
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 3000, inject=True)
    grid = gg.GGrid(g, 64, max_objects=3000)
    hist = []
    for r in range(6):
        for _ in range(3):
            u = walk.ticks(2)
            hist.append(u)
            grid.ingest(u)
        q = synth.queries(g, 200, seed=900 + r)
        _assert_same(grid.knn(q, 8), _oracle(g, np.concatenate(hist), q, 8), f"kernel {kernel} round {r}")
    grid.close()


@pytest.mark.parametrize("case", ["many_winners", "long_chains"])
def test_flush_warp_overflow_cells(gg, case, monkeypatch):
    """The warp-per-cell flush leaves a cell with more winners than it stages (WW = 128: 4096-vertex
    cells of ~500 objects) or more extents than it walks (XW = 32: 40 batches between queries) to
    the CTA kernel's overflow pass; cells of both kinds and ordinary ones in one flush, every round
    the oracle's answer, and the cleaned cells the oracle's snapshot."""
    monkeypatch.setenv("GGRID_FLUSH_KERNEL", "3")
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 2000, inject=True)
    cs = 4096 if case == "many_winners" else 128
    grid = gg.GGrid(g, cs, max_objects=2000)
    hist = []
    for r in range(3):
        for _ in range(40 if case == "long_chains" else 2):
            u = walk.ticks(1)
            if case == "long_chains":
                u = u[:300]
            hist.append(u)
            grid.ingest(u)
        q = synth.queries(g, 150, seed=1200 + r)
        _assert_same(grid.knn(q, 9), _oracle(g, np.concatenate(hist), q, 9), f"{case} round {r}")
    grid.flush_all()
    vcell = grid.vertex_cell()
    rows = []
    for c in range(grid.stats()["n_cells"]):
        o, e, d = grid.cell_objects(c)
        assert np.all(vcell[g["src"][e]] == c)
        rows += list(zip(o.tolist(), e.tolist(), d.tolist()))
    ids, e, d = oracle.snapshot_objects(np.concatenate(hist))
    assert sorted(rows) == sorted(zip(ids.tolist(), e.tolist(), d.tolist()))
    grid.close()


@pytest.mark.parametrize("k", [1, 10, 31, 32])
def test_one_warp_candidate_sort_both_paths(gg, k):
    """The one-warp level's final candidate sort runs in registers (one candidate per lane) when a
    query harvested at most 32 candidates and k <= 32, else in shared memory: objects stacked 24 at
    a time on a few hundred arcs (plus a uniform background) give queries on both sides of 32
    harvested candidates, with ties at equal offsets.  Every row the oracle's."""
    g = synth.table_ii_graph("NY", scale=0.2)
    rng = np.random.default_rng(21)
    hot = rng.choice(len(g["src"]), 250, replace=False)
    arc_c = np.repeat(hot, 24)
    off_c = (rng.integers(0, 3, len(arc_c)) * (g["w"][arc_c] // 3)).astype(np.int64)  # ties
    arc_b, off_b = synth.random_locations(g, 2000, rng)
    arc = np.concatenate([arc_c, arc_b]).astype(np.int64)
    off = np.minimum(np.concatenate([off_c, off_b]).astype(np.int64), g["w"][arc].astype(np.int64) - 1)
    n = len(arc)
    upd = np.stack([rng.permutation(n), arc, off, np.full(n, 5, np.int64)], 1).astype(np.uint32)
    q = synth.queries(g, 1200, seed=91)
    grid = gg.GGrid(g, 256, max_objects=n)
    grid.ingest(upd)
    _assert_same(grid.knn(q, k), _oracle(g, upd, q, k), f"k={k}")
    grid.close()
