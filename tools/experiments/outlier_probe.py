"""Diagnostics: the latency of the rare queries that overflow the level-0 capacity (promoted).

Replays bench.py's e2e stream on C1 (same seeds), then answers one step's queries one at a
time (Q=1) and reports the slowest ones with their promotion counts and expansion work, and the
batch time of that step with and without those queries.

    python tools/outlier_probe.py [--step 13]
"""
import argparse
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--step", type=int, default=13)
ap.add_argument("--top", type=int, default=8)
args = ap.parse_args()

cfg = synth.CONFIGS["C1"]
g = synth.config_graph("C1")
walk = synth.RandomWalk(g, cfg["n_objects"])
Q, k = cfg["n_queries"], cfg["k"]
grid = gg.GGrid(g, cfg["cell_size"], max_objects=cfg["n_objects"], async_ingest=True, profile=1)
o = torch.empty((Q, k), dtype=torch.int32, device="cuda")
d = torch.empty_like(o)
qs = None
for s in range(args.step + 1):
    u = torch.from_numpy(walk.ticks(cfg["updates_per_object"]).view(np.int32)).cuda()
    q = torch.from_numpy(synth.queries(g, Q, seed=synth.SEED_QUERIES + 10_000 + s).view(np.int32)).cuda()
    grid.ingest(u)
    if s < args.step:
        st0 = grid.stats()
        grid.knn(q, k, o, d)
        st1 = grid.stats()
        print(f"step {s}: promotions {st1['expand_promotions'] - st0['expand_promotions']}")
    qs = q
grid.flush_all()
# batch time of the step's queries
torch.cuda.synchronize()
grid.stats_reset()
st0 = grid.stats()
grid.knn(qs, k, o, d)
st1 = grid.stats()
print("batch: kernel ms", {a: round(b, 4) for a, b in st1["kernel_ms"].items() if b},
      "promotions", st1["expand_promotions"] - st0["expand_promotions"])
# one at a time
o1 = torch.empty((1, k), dtype=torch.int32, device="cuda")
d1 = torch.empty_like(o1)
res = []
for i in range(Q):
    a = grid.stats()
    t0 = time.perf_counter()
    grid.knn(qs[i:i + 1], k, o1, d1)
    t1 = time.perf_counter()
    b = grid.stats()
    res.append((t1 - t0, i, b["expand_promotions"] - a["expand_promotions"],
                b["expand_iterations"] - a["expand_iterations"], b["expand_vertices"] - a["expand_vertices"],
                {kk: round(b["kernel_ms"][kk] - a["kernel_ms"][kk], 4) for kk in ("expand", "expand_big")}))
res.sort(reverse=True)
lat = np.array([r[0] for r in res]) * 1e6
print(f"single-query wall us: median {np.median(lat):.0f}  p99 {np.percentile(lat, 99):.0f}  max {lat[0]:.0f}")
for r in res[:args.top]:
    print(f"  q{r[1]}: {1e6 * r[0]:.0f} us, promotions {r[2]}, rounds {r[3]}, vertices {r[4]}, kernel ms {r[5]}")
