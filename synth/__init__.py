"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This module holds NO arithmetic of the method (no snapshot, no distance, no
selection): it only draws road graphs, objects, location-update streams and
queries with the shapes of the paper's workloads:

* road graphs shaped like the DIMACS networks of Table II (P@55786-56221):
  a jittered, connected, planar lattice with twin arcs, integer weights
  w = max(1, round(Euclidean length)) — the paper uses 4-byte integers (P@59405);
* moving objects uniform over arcs, offset U[0, w) (message m = <o,e,d,t>, P@10382);
* a MOTO-like random walk (P@57732): every object reports once per tick in a
  random order (f = 1, P@58136); t = tick*1000 + U[0,999]; optional late and
  duplicate timestamps for the (t, seq) tie-break reading;
* queries q = <e, d> uniform over arcs (P@57873, P@45698).

Layout conventions (identical for every consumer):
  graph  : dict(n_vertices, src, dst, w, x, y)  — uint32 arrays of length n_arcs
           (x, y int32 of length n_vertices); arcs 2i and 2i+1 are twins.
  updates: uint32 array of shape (n, 4) — columns (obj, edge, offset, t); the
           arrival order is the row order (seq = global row index).
  queries: uint32 array of shape (n, 2) — columns (edge, offset).
"""
from __future__ import annotations

import json
import math
import os

import numpy as np

SEED_GRAPH, SEED_OBJECTS, SEED_UPDATES, SEED_QUERIES = 1, 2, 3, 4

# Table II shapes (P@55786-56221): |V| and directed-arc counts.
TABLE_II = {
    "NY": (264_346, 733_846),
    "COL": (435_666, 1_057_066),
    "FLA": (1_070_376, 2_712_798),
    "CAL": (1_890_815, 4_657_742),
    "LKS": (2_758_119, 6_885_658),
    "USA": (23_974_347, 58_333_344),
}

# BASELINE.json configs.
CONFIGS = {
    "C0": dict(graph="lattice32", n_objects=100, updates_per_object=10, n_queries=100, k=3, cell_size=64),
    "C1": dict(graph="NY", n_objects=10_000, updates_per_object=100, n_queries=10_000, k=10, cell_size=1024),
    "C2": dict(graph="FLA", n_objects=100_000, updates_per_object=10, n_queries=10_000, k=50, cell_size=1024),
    "C3": dict(graph="USA", n_objects=1_000_000, updates_per_object=64, n_queries=1 << 16, k=10, cell_size=1024),
}
# The bench step of each config: `preload_ticks` ticks of the walk cached once before the timed
# region (C3: 64 cached records per object = 64M records >> L2), then per step
# `step_ticks` ticks (every object reports once per tick: f = 1, P@58136) and n_queries queries.
BENCH_STEPS = {
    "C0": dict(preload_ticks=0, step_ticks=10),
    "C1": dict(preload_ticks=0, step_ticks=100),
    "C2": dict(preload_ticks=0, step_ticks=10),
    "C3": dict(preload_ticks=64, step_ticks=1),
}


def _twin_arrays(ea, eb):
    """Expand undirected edges (ea[i], eb[i]) into twin arcs 2i: a->b, 2i+1: b->a."""
    m = len(ea)
    src = np.empty(2 * m, np.uint32)
    dst = np.empty(2 * m, np.uint32)
    src[0::2], dst[0::2] = ea, eb
    src[1::2], dst[1::2] = eb, ea
    return src, dst


def lattice_graph(width: int, height: int, wmin: int = 1, wmax: int = 4, seed: int = SEED_GRAPH,
                  uniform_weight: int | None = None):
    """Full 4-neighbour width x height lattice with twin arcs (C0: 32x32 -> 1024 V, 3968 arcs).

    Vertex id = y*width + x, coordinates (x*1000, y*1000).  Undirected edge weights are
    U{wmin..wmax} (ties on purpose) or `uniform_weight` for the closed-form pin.
    """
    rng = np.random.default_rng(seed)
    ids = np.arange(width * height, dtype=np.int64).reshape(height, width)
    ha, hb = ids[:, :-1].ravel(), ids[:, 1:].ravel()
    va, vb = ids[:-1, :].ravel(), ids[1:, :].ravel()
    ea = np.concatenate([ha, va]).astype(np.uint32)
    eb = np.concatenate([hb, vb]).astype(np.uint32)
    if uniform_weight is not None:
        we = np.full(len(ea), uniform_weight, np.uint32)
    else:
        we = rng.integers(wmin, wmax + 1, size=len(ea)).astype(np.uint32)
    src, dst = _twin_arrays(ea, eb)
    w = np.repeat(we, 2)
    yy, xx = np.divmod(np.arange(width * height), width)
    return dict(n_vertices=width * height, src=src, dst=dst, w=w,
                x=(xx * 1000).astype(np.int32), y=(yy * 1000).astype(np.int32))


def road_graph(n_vertices: int, n_arcs: int, seed: int = SEED_GRAPH):
    """DIMACS-shaped planar road graph (SURVEY §8(d) 'Graph generator').

    Vertices on a ceil(sqrt(V))-wide lattice, coordinates jittered +-0.3 cell and
    scaled x1000.  Connected by construction: every row path plus one random
    vertical per adjacent row pair, then random extra verticals until the arc
    count hits `n_arcs` (twin arcs, so n_arcs must be even).
    """
    assert n_arcs % 2 == 0
    rng = np.random.default_rng(seed)
    V = int(n_vertices)
    W = int(math.ceil(math.sqrt(V)))
    rows = (V + W - 1) // W
    idx = np.arange(V, dtype=np.int64)
    r, c = np.divmod(idx, W)
    fx = (c + rng.uniform(-0.3, 0.3, V)) * 1000.0
    fy = (r + rng.uniform(-0.3, 0.3, V)) * 1000.0
    # row edges (i, i+1) inside a row
    rmask = (c[:-1] < W - 1)
    ra = idx[:-1][rmask]
    rb = ra + 1
    # vertical candidates (i, i+W)
    cand = idx[: max(V - W, 0)]
    n_edges = n_arcs // 2
    need = n_edges - len(ra)
    assert 0 <= need <= len(cand), (need, len(cand))
    # one mandatory vertical per adjacent row pair (connectivity)
    chosen = np.zeros(len(cand), bool)
    for rr in range(rows - 1):
        top = rr * W
        lim = min(W, V - (rr + 1) * W)  # columns that exist in row rr+1
        chosen[top + int(rng.integers(0, lim))] = True
    rest = np.flatnonzero(~chosen)
    extra = need - int(chosen.sum())
    assert extra >= 0
    pick = rng.choice(rest, size=extra, replace=False) if extra > 0 else np.empty(0, np.int64)
    chosen[pick] = True
    va = cand[chosen]
    vb = va + W
    ea = np.concatenate([ra, va])
    eb = np.concatenate([rb, vb])
    length = np.hypot(fx[ea] - fx[eb], fy[ea] - fy[eb])
    we = np.maximum(1, np.rint(length)).astype(np.uint32)
    src, dst = _twin_arrays(ea.astype(np.uint32), eb.astype(np.uint32))
    return dict(n_vertices=V, src=src, dst=dst, w=np.repeat(we, 2),
                x=np.rint(fx).astype(np.int32), y=np.rint(fy).astype(np.int32))


def table_ii_graph(name: str, seed: int = SEED_GRAPH, scale: float = 1.0):
    """Road graph with the |V| / arc counts of a Table II network (optionally scaled down)."""
    V, A = TABLE_II[name]
    if scale != 1.0:
        V = max(16, int(V * scale))
        A = 2 * int(A / 2 * scale)
    return road_graph(V, A, seed)


def config_graph(cfg: str, seed: int = SEED_GRAPH):
    name = CONFIGS[cfg]["graph"]
    if name == "lattice32":
        return lattice_graph(32, 32, 1, 4, seed)
    return table_ii_graph(name, seed)


def out_csr(graph):
    """Out-arc adjacency (generator-side helper for the random walk only)."""
    src = graph["src"].astype(np.int64)
    order = np.argsort(src, kind="stable").astype(np.int64)
    deg = np.bincount(src, minlength=graph["n_vertices"])
    ptr = np.zeros(graph["n_vertices"] + 1, np.int64)
    np.cumsum(deg, out=ptr[1:])
    return ptr, order


def random_locations(graph, n: int, rng):
    """n uniform locations (arc, offset) with 0 <= offset < w(arc)."""
    A = len(graph["src"])
    arc = rng.integers(0, A, size=n).astype(np.int64)
    off = (rng.random(n) * graph["w"][arc]).astype(np.int64)
    off = np.minimum(off, graph["w"][arc].astype(np.int64) - 1)
    return arc.astype(np.uint32), off.astype(np.uint32)


def queries(graph, n: int, seed: int = SEED_QUERIES):
    """n queries (edge, offset), uniform arc, U[0,w) offset (P@57873)."""
    rng = np.random.default_rng(seed)
    arc, off = random_locations(graph, n, rng)
    return np.stack([arc, off], axis=1).astype(np.uint32)


class RandomWalk:
    """MOTO-like random walk of n objects on `graph` (SURVEY §8(d) 'Updates').

    Each tick every object advances U[10,30] length units along its arc, turning onto a
    random non-U-turn out-arc at each vertex (U-turn only at dead ends), and reports
    once, in a random order.  t = tick*1000 + U[0,999].  With `inject`, ~2% of the
    reports repeat the object's previous t (duplicate) and ~2% are late
    (t - U{1..3}*1000), exercising the (t, seq) reading S7/S8.
    """

    def __init__(self, graph, n_objects: int, seed_objects: int = SEED_OBJECTS,
                 seed_updates: int = SEED_UPDATES, inject: bool = False, speed=(10, 30),
                 obj_ids=None):
        self.g = graph
        self.n = int(n_objects)
        self.w = graph["w"].astype(np.int64)
        self.dst = graph["dst"].astype(np.int64)
        self.ptr, self.order = out_csr(graph)
        rng0 = np.random.default_rng(seed_objects)
        arc, off = random_locations(graph, self.n, rng0)
        self.arc = arc.astype(np.int64)
        self.off = off.astype(np.int64)
        self.rng = np.random.default_rng(seed_updates)
        self.tick_no = 0
        self.inject = inject
        self.speed = speed
        self.prev_t = np.zeros(self.n, np.int64)
        self.obj_ids = (np.arange(self.n, dtype=np.uint32) if obj_ids is None
                        else np.asarray(obj_ids, np.uint32))

    def _advance(self):
        rng = self.rng
        self.off += rng.integers(self.speed[0], self.speed[1] + 1, size=self.n)
        over = np.flatnonzero(self.off >= self.w[self.arc])
        while len(over):
            a = self.arc[over]
            self.off[over] -= self.w[a]
            v = self.dst[a]
            deg = self.ptr[v + 1] - self.ptr[v]
            twin = a ^ 1
            j = (rng.random(len(over)) * np.maximum(deg - 1, 1)).astype(np.int64)
            j = np.minimum(j, np.maximum(deg - 2, 0))
            cand = self.order[self.ptr[v] + j]
            last = self.order[self.ptr[v] + deg - 1]
            cand = np.where((deg > 1) & (cand == twin), last, cand)
            cand = np.where(deg == 1, self.order[self.ptr[v]], cand)
            self.arc[over] = cand
            over = over[self.off[over] >= self.w[self.arc[over]]]

    def tick(self):
        """One tick: returns uint32 (n, 4) updates (obj, edge, offset, t) in arrival order."""
        self._advance()
        rng = self.rng
        t = self.tick_no * 1000 + rng.integers(0, 1000, size=self.n)
        if self.inject and self.tick_no > 0:
            u = rng.random(self.n)
            dup = u < 0.02
            late = (u >= 0.02) & (u < 0.04)
            t = np.where(dup, self.prev_t, t)
            t = np.where(late, np.maximum(0, t - 1000 * rng.integers(1, 4, size=self.n)), t)
        self.prev_t = t
        perm = rng.permutation(self.n)
        out = np.empty((self.n, 4), np.uint32)
        out[:, 0] = self.obj_ids[perm]
        out[:, 1] = self.arc[perm]
        out[:, 2] = self.off[perm]
        out[:, 3] = t[perm]
        self.tick_no += 1
        return out

    def ticks(self, n_ticks: int):
        if n_ticks == 0:
            return np.empty((0, 4), np.uint32)
        return np.concatenate([self.tick() for _ in range(n_ticks)])


def golden_path(name: str) -> str:
    return os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden", name)


def fig1_fixture():
    """The builder-authored Fig. 1 fixture (tests/golden/fig1.json; the figure's map is
    absent from PAPER.md, only the query point <8.5,6.5> and the answer <o5,o2,o4> survive,
    P@2932-3378)."""
    with open(golden_path("fig1.json")) as f:
        d = json.load(f)
    W, H = d["lattice"]["width"], d["lattice"]["height"]
    g = lattice_graph(W, H, uniform_weight=d["lattice"]["weight"])
    return d, g
