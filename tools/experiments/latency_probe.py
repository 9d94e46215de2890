"""Single-query (Q=1) latency breakdown on C1: per-kernel device time per ggrid_knn call."""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402

g = synth.config_graph("C1")
walk = synth.RandomWalk(g, 10_000)
grid = gg.GGrid(g, 1024, max_objects=10_000, profile=True)
grid.ingest(walk.ticks(100))
grid.flush_all()
q = torch.from_numpy(synth.queries(g, 200, seed=77).view(np.int32)).cuda()
o = torch.empty((1, 10), dtype=torch.int32, device="cuda")
d = torch.empty_like(o)
for i in range(20):
    grid.knn(q[i:i + 1], 10, o, d)
grid.stats_reset()
s0 = grid.stats()
N = 100
t0 = time.perf_counter()
for i in range(N):
    grid.knn(q[100 + i % 100:101 + i % 100], 10, o, d)
t1 = time.perf_counter()
s1 = grid.stats()
print(f"host wall per call {1e6 * (t1 - t0) / N:.1f} us; rounds/call {(s1['knn_rounds'] - s0['knn_rounds']) / N:.2f}")
for kind, ms in s1["kernel_ms"].items():
    n = s1["kernel_launches"][kind]
    if n:
        print(f"  {kind:16s} {n / N:5.2f} launches/call  {1e3 * ms / N:8.1f} us/call")
w = {k: (s1[k] - s0[k]) / N for k in ("expand_iterations", "expand_vertices", "expand_arcs", "expand_objects")}
print("work/query", w)
