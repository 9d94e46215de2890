"""The ingest paths (opts.ingest_kernels) against the oracle (-m gpu).

Alg. 1 (P@18177-19248) caches each message in the log of cell(src(e)); the index state it
leaves must be the same whichever launch structure builds it: a single cooperative launch
(classify / extent allocation / scatter separated by grid barriers) in its cell-hash variant
(ingest_kernels=1) or its direct variant (one rank atomic per update, ingest_kernels=2) --
the default picks one for a batch that fits one resident wave -- or the three-launch path
(ingest_kernels=3; also the default's fallback for larger batches).  Bit-exact: cleaned cells equal the oracle's latest-per-object
snapshot, kNN rows equal the full-Dijkstra oracle's.
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


def _cells(grid, g):
    vcell = grid.vertex_cell()
    rows = []
    for c in range(grid.stats()["n_cells"]):
        o, e, d = grid.cell_objects(c)
        assert np.all(vcell[g["src"][e]] == c)
        rows += list(zip(o.tolist(), e.tolist(), d.tolist()))
    return sorted(rows)


def _same(got, ref, msg):
    assert np.array_equal(got[0], ref[0]) and np.array_equal(got[1], ref[1]), msg


@pytest.mark.parametrize("mode", [0, 1, 2, 3, 4])
def test_ingest_paths_same_state(gg, mode):
    """Multi-CTA batches (300k updates over a 53k-vertex graph, 207 cells of 256 vertices);
    a batch with one bad record in its middle is rejected whole by both paths."""
    g = synth.table_ii_graph("NY", scale=0.2)
    upd = synth.RandomWalk(g, 20_000, inject=True).ticks(30)
    half = len(upd) // 2
    grid = gg.GGrid(g, 256, max_objects=20_000, ingest_kernels=mode)
    grid.ingest(upd[:half])
    bad = upd[half:].copy()
    bad[len(bad) // 2, 1] = len(g["src"])
    with pytest.raises(gg.GGridError) as e:
        grid.ingest(bad)
    assert e.value.rc == gg.GGRID_EINVAL
    grid.ingest(upd[half:])
    st = grid.stats()
    assert st["n_updates"] == len(upd)
    if mode in (3, 4):
        assert st["kernel_launches"]["ingest_alloc"] == 3
    else:
        assert st["kernel_launches"]["ingest_alloc"] == 0  # one launch per batch
    q = synth.queries(g, 400)
    _same(grid.knn(q, 10), oracle.knn_from_updates(g, upd, q, 10), f"mode {mode}")
    grid.flush_all()
    ids, e_, d_ = oracle.snapshot_objects(upd)
    assert _cells(grid, g) == sorted(zip(ids.tolist(), e_.tolist(), d_.tolist()))
    grid.close()


def test_fused_fallback_beyond_one_wave(gg):
    """A batch larger than one resident wave (> 8,192 updates per SM) takes the three-launch
    path under the default mode; a batch whose tiles meet more distinct cells than the shared
    cell hash holds (cell_size 1: every vertex a cell) does too.  Both exact."""
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 4000, inject=True)
    upd = walk.ticks(400)  # 1.6M updates
    grid = gg.GGrid(g, 64, max_objects=4096)
    grid.ingest(upd)
    assert grid.stats()["kernel_launches"]["ingest_alloc"] == 1
    q = synth.queries(g, 200)
    _same(grid.knn(q, 8), oracle.knn_from_updates(g, upd, q, 8), "beyond one wave")
    grid.close()
    small = walk.ticks(200)  # 800k updates over 13k single-vertex cells
    grid = gg.GGrid(g, 1, max_objects=4096)
    grid.ingest(small)  # (whichever path the plan picks for a tile meeting ~5k distinct cells)
    _same(grid.knn(q, 8), oracle.knn_from_updates(g, small, q, 8), "cell_size 1")
    grid.close()


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_fused_many_small_batches(gg, mode):
    """Single-update and tiny batches (one CTA, grid barrier of one) interleaved with queries."""
    g = synth.lattice_graph(16, 16, 1, 4)
    walk = synth.RandomWalk(g, 50, inject=True)
    grid = gg.GGrid(g, 16, max_objects=64, ingest_kernels=mode)
    hist = []
    for r in range(6):
        u = walk.ticks(1)
        for i in range(0, len(u), 7):
            grid.ingest(u[i:i + 7])
        grid.ingest(u[:1])  # a duplicate (same t, later seq) of an earlier record
        hist += [u, u[:1]]
        q = synth.queries(g, 40, seed=300 + r)
        _same(grid.knn(q, 4), oracle.knn_from_updates(g, np.concatenate(hist), q, 4), f"round {r}")
    assert grid.stats()["kernel_launches"]["ingest_alloc"] == 0
    grid.close()


# ------------------------------------------------------------------ stream order of caller inputs
def _poisoned_then_valid(torch, dst, src, stream, spin_cycles):
    """dst is first filled with invalid records (edge = 2^32-1) synchronously; then, queued on
    `stream` behind a spin kernel, overwritten with the valid batch src.  A library call that
    read dst before the copy ran would see the invalid records (EINVAL) -- the race of the
    round-1 C4 sweep (tools/c4_sweep.py)."""
    dst.fill_(-1)
    torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        torch.cuda._sleep(spin_cycles)
        dst.copy_(src)


@pytest.mark.parametrize("producer", ["side_stream", "default_stream"])
def test_device_input_ordered_after_producer(gg, producer):
    """50 ingests of a 10^6-row device batch produced by still-running torch work, with no
    host synchronisation between producing and ingesting: every batch is accepted and the
    answers are the oracle's (ggrid_wait_stream / the legacy-stream ordering of the C ABI)."""
    import torch

    g = synth.table_ii_graph("NY", scale=0.2)
    walk = synth.RandomWalk(g, 20_000)
    grid = gg.GGrid(g, 256, max_objects=20_000, log_capacity=1 << 26)
    side = torch.cuda.Stream() if producer == "side_stream" else torch.cuda.default_stream()
    dev = torch.empty((1_000_000, 4), dtype=torch.int32, device="cuda")
    hist = []
    for it in range(50):
        u = walk.ticks(50)  # 10^6 updates
        hist.append(u)
        src = torch.from_numpy(u.view(np.int32)).cuda()
        _poisoned_then_valid(torch, dev, src, side, 2_000_000)
        with torch.cuda.stream(side):
            grid.ingest(dev)  # no synchronize: the library must wait for the copy
    torch.cuda.synchronize()
    q = synth.queries(g, 300)
    _same(grid.knn(q, 10), oracle.knn_from_updates(g, np.concatenate(hist), q, 10), producer)
    grid.close()


def test_async_ingest_input_reuse_after_signal(gg):
    """opts.async_ingest: the kernels of an ingest read the device batch after the call
    returns.  The binding orders the caller's stream after them (ggrid_signal_stream), so the
    caller may overwrite the buffer right away; answers stay the oracle's."""
    import torch

    g = synth.table_ii_graph("NY", scale=0.1)
    walk = synth.RandomWalk(g, 5_000)
    grid = gg.GGrid(g, 256, max_objects=5_000, async_ingest=True)
    dev = torch.empty((200_000, 4), dtype=torch.int32, device="cuda")
    hist = []
    for it in range(20):
        u = walk.ticks(40)
        hist.append(u)
        dev.copy_(torch.from_numpy(u.view(np.int32)))
        grid.ingest(dev)
        dev.fill_(-1)  # queued after the library's kernels on the caller's (current) stream
    grid.sync()
    q = synth.queries(g, 200)
    _same(grid.knn(q, 8), oracle.knn_from_updates(g, np.concatenate(hist), q, 8), "async reuse")
    grid.close()


@pytest.mark.parametrize("mode", [0, 1, 2, 3, 4])
def test_rejected_batch_leaves_t_now(gg, mode):
    """A rejected batch changes no observable state (ggrid.h): its valid records' far-future
    t must not become t_now of the expiry rule (reading R21), which would expire every cached
    extent of an index built with t_delta."""
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 2_000)
    grid = gg.GGrid(g, 64, max_objects=2_000, t_delta=50_000, ingest_kernels=mode)
    upd = walk.ticks(20)
    grid.ingest(upd)
    t_now = grid.stats()["t_now"]
    bad = walk.ticks(2).copy()
    bad[:, 3] = 4_000_000_000
    bad[len(bad) // 3, 2] = 0xFFFFFFF0  # one offset out of range: the batch is rejected
    with pytest.raises(gg.GGridError) as e:
        grid.ingest(bad)
    assert e.value.rc == gg.GGRID_EINVAL
    assert grid.stats()["t_now"] == t_now
    q = synth.queries(g, 200)
    _same(grid.knn(q, 6), oracle.knn_from_updates(g, upd, q, 6), "after a rejected batch")
    assert grid.stats()["records_expired"] == 0
    grid.close()


def test_sustained_stream_beyond_2_32_updates(gg):
    """A handle takes more than 2^32 updates (a sustained stream): the 32-bit
    arrival index is re-based at a garbage collection and the answers stay the oracle's.
    Two device batches A, B (10^7 updates each) alternate 215 times (4.3e9 updates, ending
    with B); by max-(t, arrival) the final snapshot equals the oracle's snapshot of [A, B]
    (repeating a batch adds no t value, and the last copy of each holds every record's latest
    arrival)."""
    import torch

    g = synth.table_ii_graph("NY")
    walk = synth.RandomWalk(g, 100_000, inject=True)
    a, b = walk.ticks(100), walk.ticks(100)
    da = torch.from_numpy(a.view(np.int32)).cuda()
    db = torch.from_numpy(b.view(np.int32)).cuda()
    grid = gg.GGrid(g, 1024, max_objects=100_000, log_capacity=1 << 26)
    q = synth.queries(g, 500)
    for it in range(215):
        grid.ingest(da)
        grid.ingest(db)
        if it == 3:  # before the re-base: answers of the stream so far
            _same(grid.knn(q, 10), oracle.knn_from_updates(g, np.concatenate([a, b]), q, 10), "before")
    st = grid.stats()
    assert st["n_updates"] == 430 * len(a) > (1 << 32)
    assert st["seq_rebases"] == 1
    _same(grid.knn(q, 10), oracle.knn_from_updates(g, np.concatenate([a, b]), q, 10), "after the re-base")
    # ties across the re-base: a batch re-sent after it still wins equal timestamps
    grid.ingest(da)
    _same(grid.knn(q, 10), oracle.knn_from_updates(g, np.concatenate([b, a]), q, 10), "A re-sent")
    grid.close()


def test_overflowing_batch_is_eoverflow(gg):
    """A single batch of 2^32 - 1 updates cannot be ordered by a 32-bit arrival index (ggrid.h):
    EOVERFLOW, checked before the buffer is read."""
    import torch

    g = synth.lattice_graph(8, 8, 1, 4)
    grid = gg.GGrid(g, 16, max_objects=16)
    tiny = torch.zeros((1, 4), dtype=torch.int32, device="cuda")
    with pytest.raises(gg.GGridError) as e:
        gg.ggrid_ingest(grid.h, tiny, (1 << 32) - 1)
    assert e.value.rc == gg.GGRID_EOVERFLOW
    assert grid.stats()["n_updates"] == 0
    grid.close()


@pytest.mark.parametrize("extra", [0, 1])
def test_direct_launch_at_capacity(gg, extra):
    """The direct launch holds at most 2 CTAs x 512 threads x 8 updates per SM (1,212,416 on a
    148-SM B200): a batch of exactly that many updates takes it with every register slot in use,
    one more falls back to the other paths; both exact.  Single-vertex cells (many distinct cells
    per tile, the direct path's regime)."""
    import torch

    sms = torch.cuda.get_device_properties(0).multi_processor_count
    n = sms * 2 * 512 * 8 + extra
    g = synth.table_ii_graph("NY", scale=0.05)
    walk = synth.RandomWalk(g, 8000, inject=True)
    upd = walk.ticks(-(-n // 8000))[:n]
    grid = gg.GGrid(g, 1, max_objects=8000, ingest_kernels=2)
    grid.ingest(upd)
    st = grid.stats()
    assert st["kernel_launches"]["ingest_alloc"] == (1 if extra else 0)
    q = synth.queries(g, 300, seed=123)
    _same(grid.knn(q, 8), oracle.knn_from_updates(g, upd, q, 8), f"n={n}")
    grid.close()
