"""Diagnostics: per-step wall time of bench.py's pipelined e2e loop (C1), with variants that
isolate why the last steps of the loop are slow.

    python tools/e2e_tail.py [--steps 8] [--variant plain|rev|extra|sync]
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
ap.add_argument("--steps", type=int, default=8)
ap.add_argument("--variant", default="plain")
args = ap.parse_args()

g = synth.config_graph("C1")
walk = synth.RandomWalk(g, 10_000)
grid = gg.GGrid(g, 1024, max_objects=10_000, async_ingest=True)
Q, k = 10_000, 10
n = args.steps
hus = [torch.from_numpy(walk.ticks(100).view(np.int32)).pin_memory() for _ in range(3 + n + 1)]
hqs = [torch.from_numpy(synth.queries(g, Q, seed=100 + i).view(np.int32)).pin_memory() for i in range(3 + n + 1)]
if args.variant == "rev":
    hus = hus[:3] + hus[3:][::-1]
    hqs = hqs[:3] + hqs[3:][::-1]
if "warm" in args.variant:  # one DMA from every pinned buffer first
    su = torch.empty_like(hus[0], device="cuda")
    sq = torch.empty_like(hqs[0], device="cuda")
    for a, b in zip(hus, hqs):
        su.copy_(a)
        sq.copy_(b)
    torch.cuda.synchronize()
h_o = torch.empty((Q, k), dtype=torch.int32).pin_memory()
h_d = torch.empty((Q, k), dtype=torch.int32).pin_memory()
for s in range(3):
    grid.ingest_stage(hus[s])
    grid.ingest_commit()
    grid.knn(hqs[s], k, h_o, h_d)
torch.cuda.synchronize()
t0 = time.perf_counter()
ts = []
parts = []
qs = "qstage" in args.variant
grid.ingest_stage(hus[3])
if qs:
    grid.query_stage(hqs[3])
for s in range(3, 3 + n):
    a = time.perf_counter()
    grid.ingest_commit()
    b = time.perf_counter()
    if s + 1 < 3 + n or "extra" in args.variant:
        grid.ingest_stage(hus[s + 1])
        if qs:
            grid.query_stage(hqs[s + 1])
    c = time.perf_counter()
    if qs:
        grid.knn_commit(k, h_o, h_d)
    else:
        grid.knn(hqs[s], k, h_o, h_d)
    if "sync" in args.variant:
        grid.sync()
    ts.append(time.perf_counter())
    parts.append((round(1e3 * (b - a), 3), round(1e3 * (c - b), 3), round(1e3 * (ts[-1] - c), 3)))
print(args.variant, "step ms:", [round(1e3 * (b - a), 3) for a, b in zip([t0] + ts[:-1], ts)])
print("  (commit, stage, knn) ms:", parts[-4:])
