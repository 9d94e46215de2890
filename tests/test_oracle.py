"""Pins for the CPU oracle (runs under -m "not gpu").

Each test checks the oracle against something other than itself (SURVEY §8(c) table
"What pins each part"):
  * snapshot      — brute-force group-by/max on streams with late and duplicate t;
  * point distance (S1-S4) — Floyd-Warshall on the graph subdivided at every
                    object/query offset (an independent construction of the same
                    network distance), on tiny random directed graphs;
  * scale         — closed-form Manhattan distances on uniform-weight lattices and
                    scipy.sparse.csgraph.dijkstra on road-shaped graphs;
  * selection     — k >= |O| full sort, constructed ties, padding, the u32 range (S18);
  * Fig. 1        — the paper's answer <o5, o2, o4> on the builder-authored fixture.
"""
import itertools
import json

import numpy as np
import pytest

import synth

INF = float("inf")


# ----------------------------------------------------------------------------- snapshot
def _brute_latest(updates):
    best = {}
    for seq, (o, e, d, t) in enumerate(updates.tolist()):
        key = (t, seq)
        if o not in best or key > best[o][0]:
            best[o] = (key, e, d)
    return best


@pytest.mark.parametrize("seed", range(20))
def test_snapshot_matches_bruteforce(oracle_mod, seed):
    rng = np.random.default_rng(seed)
    n, n_obj = 300, 17
    u = np.zeros((n, 4), np.uint32)
    u[:, 0] = rng.integers(0, n_obj, n)
    u[:, 1] = rng.integers(0, 50, n)
    u[:, 2] = rng.integers(0, 9, n)
    u[:, 3] = rng.integers(0, 12, n)  # many equal and out-of-order timestamps
    # feed it in several batches to exercise seq0 continuity
    snap = oracle_mod.Snapshot(n_obj + 3)
    for part in np.array_split(u, 4):
        snap.apply(part)
    ids, e, d = snap.objects()
    ref = _brute_latest(u)
    assert sorted(ref) == ids.tolist()
    for i, o in enumerate(ids.tolist()):
        assert (e[i], d[i]) == ref[o][1:]
        assert (snap.t[o], snap.seq[o]) == ref[o][0]


def test_snapshot_hand_stream(oracle_mod):
    # (obj, edge, off, t): object 1 gets a late update (t=5 after t=9): t wins, not arrival;
    # object 2 gets two t=7 updates: the later arrival (higher seq) wins (reading S7/S8).
    u = np.array([[1, 10, 0, 9], [2, 20, 1, 7], [1, 11, 0, 5], [2, 21, 2, 7], [3, 30, 3, 0]], np.uint32)
    ids, e, d = oracle_mod.snapshot_objects(u)
    assert ids.tolist() == [1, 2, 3]
    assert e.tolist() == [10, 21, 30]
    assert d.tolist() == [0, 2, 3]


# ------------------------------------------------------------ Floyd-Warshall (subdivided)
def _subdivided_fw(n_v, src, dst, w, points):
    """points: list of (arc, offset).  Returns dict point -> node id and the FW matrix."""
    cuts = {a: {0, int(w[a])} for a in range(len(src))}
    for a, d in points:
        cuts[a].add(int(d))
    node = {}
    nid = n_v
    for a in range(len(src)):
        for d in sorted(cuts[a]):
            if d == 0:
                node[(a, d)] = int(src[a])
            elif d == int(w[a]):
                node[(a, d)] = int(dst[a])
            else:
                node[(a, d)] = nid
                nid += 1
    M = np.full((nid, nid), INF)
    np.fill_diagonal(M, 0)
    for a in range(len(src)):
        ds = sorted(cuts[a])
        for x, y in zip(ds[:-1], ds[1:]):
            i, j = node[(a, x)], node[(a, y)]
            M[i, j] = min(M[i, j], y - x)
    for m in range(nid):
        M = np.minimum(M, M[:, m:m + 1] + M[m:m + 1, :])
    return node, M


def _random_digraph(rng, n_v, n_a, wmax):
    src = rng.integers(0, n_v, n_a).astype(np.uint32)
    dst = rng.integers(0, n_v, n_a).astype(np.uint32)
    w = rng.integers(1, wmax + 1, n_a).astype(np.uint32)
    return dict(n_vertices=n_v, src=src, dst=dst, w=w)


@pytest.mark.parametrize("seed", range(60))
def test_knn_equals_subdivided_floyd_warshall(oracle_mod, seed):
    rng = np.random.default_rng(1000 + seed)
    n_v = int(rng.integers(2, 9))
    g = _random_digraph(rng, n_v, int(rng.integers(1, 3 * n_v + 1)), wmax=5)
    A = len(g["src"])
    n_obj = int(rng.integers(1, 10))
    oe = rng.integers(0, A, n_obj).astype(np.uint32)
    oo = (rng.random(n_obj) * g["w"][oe]).astype(np.uint32)
    if seed % 3 == 0:
        oo[: n_obj // 2] = 0  # objects on vertices -> ties
    oid = rng.permutation(100)[:n_obj].astype(np.uint32)
    nq = 6
    qe = rng.integers(0, A, nq).astype(np.uint32)
    qo = (rng.random(nq) * g["w"][qe]).astype(np.uint32)
    qo[0] = 0
    pts = [(int(a), int(d)) for a, d in zip(oe, oo)] + [(int(a), int(d)) for a, d in zip(qe, qo)]
    node, M = _subdivided_fw(n_v, g["src"], g["dst"], g["w"], pts)
    q = np.stack([qe, qo], 1)
    for k in (1, 2, n_obj, n_obj + 3):
        for mode in (oracle_mod.FULL, oracle_mod.EARLY):
            out_o, out_d = oracle_mod.knn(g, oid, oe, oo, q, k, mode=mode, threads=2)
            for i in range(nq):
                qn = node[(int(qe[i]), int(qo[i]))]
                ref = sorted((M[qn, node[(int(a), int(d))]], int(o)) for a, d, o in zip(oe, oo, oid))
                ref = [(int(dd), o) for dd, o in ref if dd < INF][:k]
                ref += [(oracle_mod.PAD, oracle_mod.PAD)] * (k - len(ref))
                got = list(zip(out_d[i].tolist(), out_o[i].tolist()))
                assert got == ref, (seed, k, mode, i)


def test_same_arc_term_needed(oracle_mod):
    """Reading S2: object ahead of q on q's own arc (no cycle back) is at d_o - d_q."""
    g = dict(n_vertices=2, src=np.array([0], np.uint32), dst=np.array([1], np.uint32),
             w=np.array([10], np.uint32))
    out_o, out_d = oracle_mod.knn(g, [7, 8], [0, 0], [6, 2], np.array([[0, 4]]), 2)
    # object 7 is 2 ahead; object 8 is behind q and unreachable (no path back to vertex 0)
    assert out_o.tolist() == [[7, oracle_mod.PAD]]
    assert out_d.tolist() == [[2, oracle_mod.PAD]]


def test_u32_distance_range(oracle_mod):
    """Reading S18: distances are u32; >= 2^32-1 means unreachable."""
    big = 1 << 31
    g = dict(n_vertices=3, src=np.array([0, 1], np.uint32), dst=np.array([1, 2], np.uint32),
             w=np.array([big, big], np.uint32))
    out_o, out_d = oracle_mod.knn(g, [1, 2, 3], [1, 1, 0], [big - 2, big - 1, 5], np.array([[0, 0]]), 3)
    assert out_o.tolist() == [[3, 1, oracle_mod.PAD]]
    assert out_d.tolist() == [[5, (1 << 32) - 2, oracle_mod.PAD]]


def test_ties_broken_by_id(oracle_mod):
    g = synth.lattice_graph(3, 3, uniform_weight=2)
    # four objects at the very same location and one equidistant elsewhere
    oid = np.array([9, 4, 6, 2, 5], np.uint32)
    oe = np.array([0, 0, 0, 0, 2], np.uint32)
    oo = np.array([1, 1, 1, 1, 1], np.uint32)
    q = np.array([[0, 0]], np.uint32)
    out_o, out_d = oracle_mod.knn(g, oid, oe, oo, q, 3)
    assert out_o.tolist() == [[2, 4, 6]]
    assert out_d.tolist() == [[1, 1, 1]]


# ------------------------------------------------------------------- lattice closed form
def _lattice_closed_form(W, c, src, dst, qa, qd, oa, od):
    def xy(v):
        return v % W, v // W

    def man(a, b):
        (ax, ay), (bx, by) = xy(a), xy(b)
        return abs(ax - bx) + abs(ay - by)

    if qd == 0:
        d1 = c * man(src[qa], src[oa]) + od
    else:
        d1 = (c - qd) + c * man(dst[qa], src[oa]) + od
    if oa == qa and od >= qd:
        d1 = min(d1, od - qd)
    return d1


@pytest.mark.parametrize("W,H,c", [(2, 2, 1), (5, 3, 3), (7, 7, 5), (40, 30, 4)])
def test_lattice_closed_form(oracle_mod, W, H, c):
    g = synth.lattice_graph(W, H, uniform_weight=c)
    rng = np.random.default_rng(W * 100 + H)
    A = len(g["src"])
    n_obj = 60
    oe = rng.integers(0, A, n_obj).astype(np.uint32)
    oo = rng.integers(0, c, n_obj).astype(np.uint32)
    oid = np.arange(n_obj, dtype=np.uint32)
    nq = 40
    qe = rng.integers(0, A, nq).astype(np.uint32)
    qo = rng.integers(0, c, nq).astype(np.uint32)
    q = np.stack([qe, qo], 1)
    out_o, out_d = oracle_mod.knn(g, oid, oe, oo, q, n_obj)
    s, d = g["src"].tolist(), g["dst"].tolist()
    for i in range(nq):
        ref = sorted((_lattice_closed_form(W, c, s, d, int(qe[i]), int(qo[i]), int(a), int(o)), int(j))
                     for j, (a, o) in enumerate(zip(oe, oo)))
        assert list(zip(out_d[i].tolist(), out_o[i].tolist())) == ref


def test_lattice_closed_form_large_early(oracle_mod):
    """A 512x512 lattice (262k vertices, ~1M arcs): EARLY and FULL against the closed form."""
    W = H = 512
    c = 7
    g = synth.lattice_graph(W, H, uniform_weight=c)
    rng = np.random.default_rng(5)
    A = len(g["src"])
    n_obj = 2000
    oe = rng.integers(0, A, n_obj).astype(np.uint32)
    oo = rng.integers(0, c, n_obj).astype(np.uint32)
    oid = rng.permutation(n_obj).astype(np.uint32)
    qe = rng.integers(0, A, 8).astype(np.uint32)
    qo = rng.integers(0, c, 8).astype(np.uint32)
    q = np.stack([qe, qo], 1)
    s, d = g["src"].tolist(), g["dst"].tolist()
    k = 10
    for mode in (oracle_mod.FULL, oracle_mod.EARLY):
        out_o, out_d = oracle_mod.knn(g, oid, oe, oo, q, k, mode=mode)
        for i in range(len(q)):
            ref = sorted((_lattice_closed_form(W, c, s, d, int(qe[i]), int(qo[i]), int(a), int(o)), int(j))
                         for j, a, o in zip(oid, oe, oo))[:k]
            assert list(zip(out_d[i].tolist(), out_o[i].tolist())) == ref


# ----------------------------------------------------------------------- scipy Dijkstra
def test_vertex_dist_matches_scipy(oracle_mod):
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import dijkstra

    g = synth.table_ii_graph("NY", scale=0.08)
    V = g["n_vertices"]
    M = csr_matrix((g["w"].astype(np.float64), (g["src"], g["dst"])), shape=(V, V))
    assert M.nnz == len(g["src"])  # no parallel arcs were merged
    rng = np.random.default_rng(3)
    for _ in range(6):
        a = int(rng.integers(0, len(g["src"])))
        d = int(rng.integers(0, g["w"][a])) if rng.random() < 0.7 else 0
        D = oracle_mod.vertex_dist(g, a, d)
        if d == 0:
            ref = dijkstra(M, indices=int(g["src"][a]))
        else:
            ref = (int(g["w"][a]) - d) + dijkstra(M, indices=int(g["dst"][a]))
        assert np.all(np.isfinite(ref))
        assert np.array_equal(D, ref.astype(np.uint64))


def test_knn_matches_scipy_objects(oracle_mod):
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import dijkstra

    g = synth.table_ii_graph("NY", scale=0.05)
    V = g["n_vertices"]
    M = csr_matrix((g["w"].astype(np.float64), (g["src"], g["dst"])), shape=(V, V))
    rng = np.random.default_rng(11)
    oe, oo = synth.random_locations(g, 500, rng)
    oid = rng.permutation(5000)[:500].astype(np.uint32)
    q = synth.queries(g, 20, seed=12)
    k = 10
    for mode in (oracle_mod.FULL, oracle_mod.EARLY):
        out_o, out_d = oracle_mod.knn(g, oid, oe, oo, q, k, mode=mode)
        for i, (qa, qd) in enumerate(q.tolist()):
            if qd == 0:
                Dv = dijkstra(M, indices=int(g["src"][qa]))
            else:
                Dv = (int(g["w"][qa]) - qd) + dijkstra(M, indices=int(g["dst"][qa]))
            dd = Dv[g["src"][oe]] + oo
            same = (oe == qa) & (oo >= qd)
            dd = np.where(same, np.minimum(dd, oo.astype(np.int64) - qd), dd)
            ref = sorted(zip(dd.astype(np.int64).tolist(), oid.tolist()))[:k]
            assert list(zip(out_d[i].tolist(), out_o[i].tolist())) == ref


def test_early_equals_full_road(oracle_mod):
    g = synth.table_ii_graph("NY", scale=0.1)
    walk = synth.RandomWalk(g, 400, inject=True)
    upd = walk.ticks(5)
    q = synth.queries(g, 64)
    for k in (1, 3, 10, 50):
        a = oracle_mod.knn_from_updates(g, upd, q, k, mode=oracle_mod.FULL)
        b = oracle_mod.knn_from_updates(g, upd, q, k, mode=oracle_mod.EARLY)
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


# ---------------------------------------------------------------------------- Fig. 1
def _arc_id(g, a, b, W):
    u = a[1] * W + a[0]
    v = b[1] * W + b[0]
    hits = np.flatnonzero((g["src"] == u) & (g["dst"] == v))
    assert len(hits) == 1
    return int(hits[0])


def test_fig1_fixture(oracle_mod):
    d, g = synth.fig1_fixture()
    W = d["lattice"]["width"]
    qa = _arc_id(g, d["query"]["from"], d["query"]["to"], W)
    ids = np.array([o["id"] for o in d["objects"]], np.uint32)
    oe = np.array([_arc_id(g, o["from"], o["to"], W) for o in d["objects"]], np.uint32)
    oo = np.array([o["offset"] for o in d["objects"]], np.uint32)
    q = np.array([[qa, d["query"]["offset"]]], np.uint32)
    out_o, out_d = oracle_mod.knn(g, ids, oe, oo, q, d["k"])
    assert out_o[0].tolist() == d["paper_answer"]  # the paper's <o5, o2, o4>
    out_o, out_d = oracle_mod.knn(g, ids, oe, oo, q, len(ids))
    assert [[int(a), int(b)] for a, b in zip(out_o[0], out_d[0])] == d["hand_order"]
    for o in d["objects"]:
        assert int(out_d[0][out_o[0].tolist().index(o["id"])]) == o["hand_dist"]
