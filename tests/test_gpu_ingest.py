"""The two ingest paths (opts.ingest_kernels) against the oracle (-m gpu).

Alg. 1 (P@18177-19248) caches each message in the log of cell(src(e)); the index state it
leaves must be the same whichever launch structure builds it: the single cooperative launch
(classify / extent allocation / scatter separated by grid barriers; default for a batch that
fits one resident wave) or the three-launch path (ingest_kernels=3; also the default's
fallback for larger batches).  Bit-exact: cleaned cells equal the oracle's latest-per-object
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


@pytest.mark.parametrize("mode", [0, 3])
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
    if mode == 0:
        assert st["kernel_launches"]["ingest_alloc"] == 0  # one launch per batch
    else:
        assert st["kernel_launches"]["ingest_alloc"] == 3
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
    grid.ingest(small)
    assert grid.stats()["kernel_launches"]["ingest_alloc"] == 1
    _same(grid.knn(q, 8), oracle.knn_from_updates(g, small, q, 8), "cell_size 1")
    grid.close()


def test_fused_many_small_batches(gg):
    """Single-update and tiny batches (one CTA, grid barrier of one) interleaved with queries."""
    g = synth.lattice_graph(16, 16, 1, 4)
    walk = synth.RandomWalk(g, 50, inject=True)
    grid = gg.GGrid(g, 16, max_objects=64)
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
