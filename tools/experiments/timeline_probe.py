"""Device timeline (CUPTI via torch.profiler) of the pipelined e2e loop of bench.py, C1."""
import os
import sys

import numpy as np
import torch
from torch.profiler import ProfilerActivity, profile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402

FRESH = "--fresh" in sys.argv
g = synth.config_graph("C1")
walk = synth.RandomWalk(g, 10_000)
grid = gg.GGrid(g, 1024, max_objects=10_000)
hus = [torch.from_numpy(walk.ticks(100).view(np.int32)).pin_memory() for _ in range(8)]
hqs = [torch.from_numpy(synth.queries(g, 10_000, seed=10 + i).view(np.int32)).pin_memory() for i in range(8)]
hq = hqs[0]
ho = torch.empty((10_000, 10), dtype=torch.int32).pin_memory()
hd = torch.empty((10_000, 10), dtype=torch.int32).pin_memory()
grid.ingest(hus[0])
grid.knn(hq, 10, ho, hd)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
    grid.ingest_stage(hus[1])
    for s in range(1, 6):
        grid.ingest_commit()
        grid.ingest_stage(hus[s + 1])
        grid.knn(hqs[s] if FRESH else hq, 10, ho, hd)
    grid.ingest_commit()
    torch.cuda.synchronize()
evs = []
for e in prof.events():
    if e.device_type == torch.autograd.DeviceType.CUDA or "cuda" in e.name.lower() or "Memcpy" in e.name:
        evs.append((e.time_range.start, e.time_range.end, e.name[:60], getattr(e, "device_type", None)))
evs.sort()
knn_t = [a for a, b, n, d in evs if n.startswith("cudaStreamWaitEvent")]
t0 = evs[0][0]
print("host wall per step (ms):", [round((b - a) / 1e3, 3) for a, b in zip(knn_t[:-1], knn_t[1:])])
for a, b, n, d in evs:
    print(f"{(a - t0):9.1f} {(b - t0):9.1f} {b - a:8.1f}  {str(d).split('.')[-1]:5s} {n}")
