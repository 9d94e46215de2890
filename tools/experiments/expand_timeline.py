"""Device timeline (CUPTI via torch.profiler) of the bench's C3 step: when the starting expansion
level and the chained level (promoted queries) start and end, i.e. the chained level's tail.

    python tools/experiments/expand_timeline.py [--steps 4] [--config C3]
"""
import argparse
import os
import sys

import numpy as np
import torch
from torch.profiler import ProfilerActivity, profile

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--config", default="C3")
args = ap.parse_args()

cfg = dict(synth.CONFIGS[args.config])
cfg.update(synth.BENCH_STEPS[args.config])
g = synth.config_graph(args.config)
n_obj, Q, k = cfg["n_objects"], cfg["n_queries"], cfg["k"]
walk = synth.RandomWalk(g, n_obj)
preload = walk.ticks(cfg["preload_ticks"]) if cfg["preload_ticks"] else None
stream = torch.cuda.Stream()
grid = gg.GGrid(g, cfg["cell_size"], max_objects=n_obj, log_capacity=1 << 28, stream=stream.cuda_stream,
                async_ingest=True)
if preload is not None:
    grid.ingest(torch.from_numpy(preload.view(np.int32)).cuda())
    grid.flush_all()
out_o = torch.empty((Q, k), dtype=torch.int32, device="cuda")
out_d = torch.empty((Q, k), dtype=torch.int32, device="cuda")
l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
inputs = []
for s in range(3 + args.steps):
    u = torch.from_numpy(walk.ticks(cfg["step_ticks"]).view(np.int32)).cuda()
    q = torch.from_numpy(synth.queries(g, Q, seed=synth.SEED_QUERIES + s).view(np.int32)).cuda()
    inputs.append((u, q))
torch.cuda.synchronize()


def step(u, q):
    torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        l2.zero_()
    grid.ingest(u)
    grid.knn(q, k, out_o, out_d)
    torch.cuda.synchronize()


for s in range(3):
    step(*inputs[s])
st0 = grid.stats()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for s in range(3, 3 + args.steps):
        step(*inputs[s])
st1 = grid.stats()
print("promoted per step", (st1["expand_promotions"] - st0["expand_promotions"]) / args.steps)
kern = sorted((e.time_range.start, e.time_range.end, e.name) for e in prof.events()
              if e.device_type == torch.autograd.DeviceType.CUDA)
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
for i, st in enumerate(steps):
    t0 = st[0][0]
    print(f"--- step {i}: span {st[-1][1] - t0:.1f} us")
    for a, b, n in st:
        print(f"  start {a - t0:8.1f}  end {b - t0:8.1f}  run {b - a:7.1f}  {n[:80]}")
