"""The prior-art comparison kernels (csrc/prior_art.cu) against the CPU
simulation of the paper's Alg. 3 (oracle/prior_art.py) and the oracle snapshot (-m gpu)."""
import json
import random

import numpy as np
import pytest

import oracle
import synth
from oracle import prior_art as pa

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


def _gpu_bundle(gg, row, eta):
    names = sorted({o for o, _ in row}, key=str)
    code = {o: i for i, o in enumerate(names)}
    obj = np.array([code[o] for o, _ in row], np.uint32)
    key = np.array([t for _, t in row], np.uint64)
    oo, ok = gg.ggrid_prior_art_bundle(obj, key, eta)
    return [(names[o], int(k)) for o, k in zip(oo, ok)]


def test_bundle_step_matches_simulation(gg):
    """Step 1 on the GPU == the simulation (reading R23) lane by lane: the W5 bundle, the
    bound-breaking mixed bundle, and random bundles at eta 4 and 5."""
    d = json.load(open(synth.golden_path("w5_xshuffle.json")))
    row = [tuple(x) for x in d["lanes"]]
    assert _gpu_bundle(gg, row, 4) == pa.x_shuffle_bundle(row, 4)
    mixed = [(0, 433), (1, 162), (1, 601), (1, 943), (0, 836), (1, 782), (1, 909), (0, 802), (0, 44), (1, 296),
             (0, 854), (1, 145), (1, 832), (0, 912), (1, 889), (0, 586)]
    assert _gpu_bundle(gg, mixed, 4) == pa.x_shuffle_bundle(mixed, 4)
    rng = random.Random(4)
    for eta in (4, 5):
        for _ in range(200):
            ts = rng.sample(range(1, 1 << 20), 2 ** eta)
            r = [(rng.randrange(rng.choice((1, 2, 4, 8))), t) for t in ts]
            assert _gpu_bundle(gg, r, eta) == pa.x_shuffle_bundle(r, eta)


@pytest.mark.parametrize("eta,bucket", [(5, 128), (4, 32), (5, 7)])
def test_prior_art_clean_locations(gg, eta, bucket):
    """write_mode 1 (until no lane is newer) collects every object's newest message: the same
    locations as the oracle snapshot; write_mode 0 (mu(eta) rounds, as printed) is counted."""
    g = synth.table_ii_graph("NY", scale=0.03)
    walk = synth.RandomWalk(g, 1500, inject=True)
    grid = gg.GGrid(g, 128, max_objects=1500)
    hist = []
    for i in range(6):
        u = walk.ticks(3)
        hist.append(u)
        grid.ingest(u)
        if i == 2:
            grid.knn(synth.queries(g, 30), 4)  # some cells with cleaned lists too
    res, e, o = grid.prior_art_clean(eta, bucket, 1, locations=True)
    ids, se, so = oracle.snapshot_objects(np.concatenate(hist), 1500)
    assert res["objects_found"] == len(ids) and res["objects_wrong"] == 0, res
    assert np.array_equal(e[ids], se) and np.array_equal(o[ids], so)
    missing = np.setdiff1d(np.arange(1500), ids)
    assert (e[missing] == gg.PAD).all()
    res0, _, _ = grid.prior_art_clean(eta, bucket, 0)
    assert res0["objects_found"] == len(ids) and res0["n_buckets"] == res["n_buckets"]
    assert res0["objects_wrong"] <= res0["objects_found"]
    grid.close()


def test_prior_art_rejects_bad_args(gg):
    g = synth.table_ii_graph("NY", scale=0.02)
    grid = gg.GGrid(g, 64, max_objects=10)
    for args in ((3, 128, 0), (5, 0, 0), (5, 128, 2)):
        with pytest.raises(gg.GGridError):
            grid.prior_art_clean(*args)
    grid.close()


# --------------------------------------------------- the paper's query pipeline (Alg. 4-6)
@pytest.mark.parametrize("graph,cs,n_obj,k,rho", [("lattice", 16, 100, 3, 1.8), ("lattice", 64, 100, 10, 1.4),
                                                   ("ny", 256, 3000, 10, 1.8), ("ny", 64, 300, 20, 3.0)])
def test_prior_art_query_pipeline_exact(gg, graph, cs, n_obj, k, rho):
    """GPU candidate cells / Bellman-Ford / first-k / unresolved vertices (Alg. 4-5, Def. 3) and
    Refine_kNN on CPU threads (Alg. 6) answer exactly what the oracle (and ggrid_knn) answers,
    under the inclusive unresolved rule (reading R13) and the same-arc term (R2): sparse objects
    (balls beyond the candidate cells) and ties (lattice weights 1..4) included."""
    g = synth.lattice_graph(32, 32, 1, 4) if graph == "lattice" else synth.table_ii_graph("NY", scale=0.05)
    upd = synth.RandomWalk(g, n_obj, inject=True).ticks(5)
    q = synth.queries(g, 300)
    grid = gg.GGrid(g, cs, max_objects=n_obj + 16)
    grid.ingest(upd)
    po, pd, res = grid.prior_art_knn(q, k, rho=rho, threads=4)
    ro, rd = oracle.knn_from_updates(g, upd, q, k)
    bad = np.flatnonzero(~((po == ro).all(1) & (pd == rd).all(1)))
    assert len(bad) == 0, f"{len(bad)} rows differ; first {bad[0]}: got {list(zip(pd[bad[0]], po[bad[0]]))} ref {list(zip(rd[bad[0]], ro[bad[0]]))}"
    go, gd = grid.knn(q, k)
    assert np.array_equal(go, po) and np.array_equal(gd, pd)
    assert res["cells"] >= len(q) and res["bf_iterations"] >= len(q) and res["threads"] == 4
    grid.close()
