"""Parity at the full sizes of BASELINE.json's larger configs (-m gpu), in the launch
configuration bench.py times.

* C3 (configs[3]): USA-shaped graph at full size (23,974,347 V / 58,333,344 arcs, Table II
  P@55786), 1M objects, 64 cached updates per object ingested in bulk batches, then steady-
  state steps of one tick (every object reports once) + 65,536 queries, k = 10, lazy flush.
* C4 (configs[4]) corners: the NY graph with |O| = 10^6 and r = 10^3 updates per query
  (10^7-update batches: the three-launch ingest path), and the FLA graph with |O| = 10^4 and
  r = 10^4 (10^8-update batches, sparse objects: large balls, higher expansion levels).

The oracle (C++, oracle/) answers sampled rows in its exact early-exit mode (cross-checked
against its full-Dijkstra mode on a few rows); the bar is bit-exact ids and distances.
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


def _check_rows(g, snap, q, go, gd, k, n_early, n_full, what):
    ids, e, d = snap.objects()
    sel = np.unique(np.concatenate([np.linspace(0, len(q) - 1, n_early).astype(np.int64),
                                    np.random.default_rng(11).choice(len(q), n_early, replace=False)]))
    ro, rd = oracle.knn(g, ids, e, d, q[sel], k, mode=oracle.EARLY)
    bad = np.flatnonzero(~((go[sel] == ro).all(1) & (gd[sel] == rd).all(1)))
    assert len(bad) == 0, (f"{what}: {len(bad)} of {len(sel)} sampled rows differ; first row {sel[bad[0]]}: "
                           f"got {list(zip(gd[sel[bad[0]]], go[sel[bad[0]]]))} ref {list(zip(rd[bad[0]], ro[bad[0]]))}")
    fo, fd = oracle.knn(g, ids, e, d, q[sel[:n_full]], k, mode=oracle.FULL)
    assert np.array_equal(fo, ro[:n_full]) and np.array_equal(fd, rd[:n_full]), f"{what}: early != full oracle"
    return len(sel)


def test_c3_full_scale_sampled(gg):
    """configs[3] at full size, bench.py's step: the bulk-ingested 64M-record log flushed lazily
    by the first query batch, then two steady-state steps; >= 256 sampled rows per step exact."""
    import torch

    g = synth.config_graph("C3")
    assert g["n_vertices"] == 23_974_347 and len(g["src"]) == 58_333_344
    n_obj = 1_000_000
    walk = synth.RandomWalk(g, n_obj)
    snap = oracle.Snapshot(n_obj)
    grid = gg.GGrid(g, 1024, max_objects=n_obj, log_capacity=1 << 27, async_ingest=True)
    for b in range(8):  # 64 ticks = 64M cached records, 8M-update batches (three-launch ingest)
        u = walk.ticks(8)
        snap.apply(u)
        grid.ingest(torch.from_numpy(u.view(np.int32)).cuda())
    k = 10
    for step in range(3):
        if step:
            u = walk.ticks(1)  # one tick: the bench's per-step update batch (fused ingest path)
            snap.apply(u)
            grid.ingest(torch.from_numpy(u.view(np.int32)).cuda())
        q = synth.queries(g, 65536, seed=synth.SEED_QUERIES + step)
        oo = torch.empty((len(q), k), dtype=torch.int32, device="cuda")
        od = torch.empty_like(oo)
        grid.knn(torch.from_numpy(q.view(np.int32)).cuda(), k, oo, od)
        go, gd = oo.cpu().numpy().view(np.uint32), od.cpu().numpy().view(np.uint32)
        assert (go[:, 0] != gg.PAD).all()
        n = _check_rows(g, snap, q, go, gd, k, 256 if step == 0 else 128, 4 if step == 0 else 1, f"C3 step {step}")
        assert n >= 256 or step > 0
    st = grid.stats()
    assert st["n_updates"] == 66 * n_obj and st["cells_flushed"] > 0
    grid.close()


def test_c4_ny_dense_objects_r1000(gg):
    """configs[4] corner: NY graph, |O| = 10^6, r = 10^3 updates per query (Q = 10^4: 10^7
    updates per step, the three-launch ingest), two steps; every row of the second step's
    batch exact (early-exit oracle) and 4 rows against full Dijkstra."""
    import torch

    from synth.device_walk import DeviceRandomWalk

    g = synth.config_graph("C1")
    n_obj, Q, k = 1_000_000, 10_000, 10
    walk = DeviceRandomWalk(g, n_obj)
    snap = oracle.Snapshot(n_obj)
    grid = gg.GGrid(g, 1024, max_objects=n_obj, log_capacity=1 << 26)
    for step in range(2):
        u = walk.ticks(10)  # 10^7 updates (device-generated)
        grid.ingest(u)
        snap.apply(u.cpu().numpy().view(np.uint32))
        q = synth.queries(g, Q, seed=synth.SEED_QUERIES + 50 + step)
        go, gd = grid.knn(q, k)
    assert grid.stats()["kernel_launches"]["ingest_alloc"] == 2  # the three-launch path, both steps
    ids, e, d = snap.objects()
    ro, rd = oracle.knn(g, ids, e, d, q, k, mode=oracle.EARLY)
    bad = np.flatnonzero(~((go == ro).all(1) & (gd == rd).all(1)))
    assert len(bad) == 0, f"C4 NY |O|=1e6 r=1e3: {len(bad)} rows differ (first {bad[0]})"
    fo, fd = oracle.knn(g, ids, e, d, q[:4], k, mode=oracle.FULL)
    assert np.array_equal(fo, go[:4]) and np.array_equal(fd, gd[:4])
    grid.close()


def test_c4_fla_sparse_objects_r10000(gg):
    """configs[4] corner: FLA graph, |O| = 10^4, r = 10^4 updates per query (Q = 10^4: 10^8
    updates per step = 10^4 ticks of 10^4 objects, device-generated); sparse objects make
    balls of ~10^3 vertices (higher expansion levels).  Sampled rows exact."""
    import torch

    from synth.device_walk import DeviceRandomWalk

    g = synth.config_graph("C2")
    n_obj, Q, k = 10_000, 10_000, 10
    walk = DeviceRandomWalk(g, n_obj)
    snap = oracle.Snapshot(n_obj)
    grid = gg.GGrid(g, 1024, max_objects=n_obj, log_capacity=(1 << 27) + (1 << 26))
    for step in range(2):
        for part in range(4):  # 4 x 2,500 ticks = 10^8 updates
            u = walk.ticks(2_500)
            grid.ingest(u)
            snap.apply(u.cpu().numpy().view(np.uint32))
            del u
        q = synth.queries(g, Q, seed=synth.SEED_QUERIES + 70 + step)
        go, gd = grid.knn(q, k)
    torch.cuda.synchronize()
    n = _check_rows(g, snap, q, go, gd, k, 256, 4, "C4 FLA |O|=1e4 r=1e4")
    assert n >= 256
    grid.close()
