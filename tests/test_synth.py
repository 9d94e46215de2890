"""Shape checks for the seeded input generators (SURVEY §8(d) recipe)."""
import numpy as np
import pytest

import synth


def test_lattice_c0_shape():
    g = synth.lattice_graph(32, 32, 1, 4)
    assert g["n_vertices"] == 1024 and len(g["src"]) == 3968  # BASELINE C0
    assert g["w"].min() >= 1 and g["w"].max() <= 4
    # twin arcs 2i / 2i+1 with equal weight (P@8380: undirected road = two arcs)
    assert np.array_equal(g["src"][0::2], g["dst"][1::2]) and np.array_equal(g["w"][0::2], g["w"][1::2])


@pytest.mark.parametrize("name", ["NY", "COL"])
def test_road_graph_table_ii_shape(name):
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import connected_components

    V, A = synth.TABLE_II[name]
    g = synth.table_ii_graph(name)
    assert g["n_vertices"] == V and len(g["src"]) == A
    assert g["src"].max() < V and g["dst"].max() < V
    assert 300 <= g["w"].min() and g["w"].max() <= 1800  # ~ 400-1,700 (jittered x1000)
    M = csr_matrix((np.ones(A), (g["src"], g["dst"])), shape=(V, V))
    assert connected_components(M, directed=True, connection="strong")[0] == 1
    # no parallel arcs
    key = g["src"].astype(np.int64) * V + g["dst"]
    assert len(np.unique(key)) == A


def test_generators_deterministic():
    g1 = synth.table_ii_graph("NY", scale=0.02)
    g2 = synth.table_ii_graph("NY", scale=0.02)
    assert all(np.array_equal(g1[k], g2[k]) for k in ("src", "dst", "w", "x", "y"))
    u1 = synth.RandomWalk(g1, 50, inject=True).ticks(4)
    u2 = synth.RandomWalk(g2, 50, inject=True).ticks(4)
    assert np.array_equal(u1, u2)


def test_random_walk_locations_valid():
    g = synth.lattice_graph(8, 8, 1, 4)  # short arcs: many vertex crossings per tick
    walk = synth.RandomWalk(g, 200, inject=True)
    u = walk.ticks(20)
    assert u.shape == (4000, 4)
    assert np.all(u[:, 2] < g["w"][u[:, 1]])
    # every tick reports every object exactly once
    for t in range(20):
        assert np.array_equal(np.sort(u[t * 200:(t + 1) * 200, 0]), np.arange(200))
    # late / duplicate injection actually happened
    t = u[:, 3].astype(np.int64).reshape(20, 200)
    assert (t[1:] < 1000 * np.arange(1, 20)[:, None]).any()


def test_queries_valid():
    g = synth.table_ii_graph("NY", scale=0.02)
    q = synth.queries(g, 1000)
    assert np.all(q[:, 1] < g["w"][q[:, 0]]) and q[:, 0].max() < len(g["src"])
