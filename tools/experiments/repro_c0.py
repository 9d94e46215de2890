"""Repro: C0 kNN at a given cell size with a forced flush kernel (debug aid)."""
import sys
import numpy as np
sys.path.insert(0, ".")
import oracle, synth
import paper_conf_icde_li0qhdy18_b200 as gg
cs = int(sys.argv[1]) if len(sys.argv) > 1 else 1
g = synth.lattice_graph(32, 32, 1, 4)
upd = synth.RandomWalk(g, 100, inject=True).ticks(10)
q = synth.queries(g, 100)
grid = gg.GGrid(g, cs, max_objects=128)
grid.ingest(upd)
for k in (1, 3, 10, 100, 130):
    o, d = grid.knn(q, k)
    ro, rd = oracle.knn_from_updates(g, upd, q, k)
    print(k, np.array_equal(o, ro) and np.array_equal(d, rd))
grid.close()
