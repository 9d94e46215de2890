"""Device timeline (CUPTI via torch.profiler) of bench.py's device-timed C1 step: where the
step's time goes (each kernel, and the idle gaps between them: host launch latency and the
library's host synchronisations).

    python tools/step_timeline.py [--steps 4] [--profile-events 0|1]
"""
import argparse
import os
import sys

import numpy as np
import torch
from torch.profiler import ProfilerActivity, profile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--profile-events", type=int, default=1)
ap.add_argument("--config", default="C1")
ap.add_argument("--async-ingest", type=int, default=1)
args = ap.parse_args()

cfg = synth.CONFIGS[args.config]
g = synth.config_graph(args.config)
walk = synth.RandomWalk(g, cfg["n_objects"])
stream = torch.cuda.Stream()
grid = gg.GGrid(g, cfg["cell_size"], max_objects=cfg["n_objects"], profile=bool(args.profile_events),
                stream=stream.cuda_stream, async_ingest=bool(args.async_ingest))
Q, k = cfg["n_queries"], cfg["k"]
out_o = torch.empty((Q, k), dtype=torch.int32, device="cuda")
out_d = torch.empty((Q, k), dtype=torch.int32, device="cuda")
l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
inputs = []
for s in range(3 + args.steps):
    u = torch.from_numpy(walk.ticks(cfg["updates_per_object"]).view(np.int32)).cuda()
    q = torch.from_numpy(synth.queries(g, Q, seed=synth.SEED_QUERIES + s).view(np.int32)).cuda()
    inputs.append((u, q))


def step(u, q, ev):
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        l2.zero_()
    e0.record(stream)
    grid.ingest(u)
    grid.knn(q, k, out_o, out_d)
    e1.record(stream)
    e1.synchronize()
    ev.append(e0.elapsed_time(e1))


ev = []
for s in range(3):
    step(*inputs[s], ev)
ev.clear()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for s in range(3, 3 + args.steps):
        step(*inputs[s], ev)
torch.cuda.synchronize()
kern = sorted((e.time_range.start, e.time_range.end, e.name) for e in prof.events()
              if e.device_type == torch.autograd.DeviceType.CUDA)
# split into steps at the L2-flush fill kernels
steps, curr = [], None
for a, b, n in kern:
    if "FillFunctor" in n:
        if curr:
            steps.append(curr)
        curr = []
        continue
    if curr is not None:
        curr.append((a, b, n))
if curr:
    steps.append(curr)
print("event ms per step:", [round(x, 4) for x in ev])
for i, st in enumerate(steps):
    t0 = st[0][0]
    busy = sum(b - a for a, b, _ in st)
    span = st[-1][1] - t0
    print(f"--- step {i}: first kernel -> last kernel end {span:.1f} us, kernel busy {busy:.1f} us, "
          f"gaps {span - busy:.1f} us")
    prev = t0
    for a, b, n in st:
        print(f"  gap {a - prev:7.1f}  run {b - a:7.1f}  {n[:70]}")
        prev = b
