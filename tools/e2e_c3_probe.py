"""Where does bench.py's end-to-end step spend its time at C3 (USA-shaped, 1M objects, 64M cached)?

Variants (wall clock per step, after warm-up, pinned host buffers):
  inplace   the bench loop: ggrid_ingest_stage / ggrid_query_stage / commit, answers written by
            the kernels straight into pinned host memory (mapped)
  devout    the same loop with device answer buffers and one torch D2H copy per step
  serial    ggrid_ingest(pinned) then ggrid_knn(pinned queries, pinned answers), no staging
and a CUPTI timeline (torch.profiler) of three steps of `inplace`.

    python tools/e2e_c3_probe.py [--steps 10] [--trace gpurun_out/e2e_c3_trace.txt]
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
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--config", default="C3")
ap.add_argument("--trace", default="")
args = ap.parse_args()

cfg = dict(synth.CONFIGS[args.config])
cfg.update(synth.BENCH_STEPS[args.config])
g = synth.config_graph(args.config)
n_obj, Q, k = cfg["n_objects"], cfg["n_queries"], cfg["k"]
walk = synth.RandomWalk(g, n_obj)
pre = walk.ticks(cfg["preload_ticks"])
N = args.steps + 3
hus = [torch.from_numpy(walk.ticks(cfg["step_ticks"]).view(np.int32)).pin_memory() for _ in range(N)]
hqs = [torch.from_numpy(synth.queries(g, Q, seed=100 + i).view(np.int32)).pin_memory() for i in range(N)]
ho = torch.empty((Q, k), dtype=torch.int32).pin_memory()
hd = torch.empty((Q, k), dtype=torch.int32).pin_memory()
do = torch.empty((Q, k), dtype=torch.int32, device="cuda")
dd = torch.empty((Q, k), dtype=torch.int32, device="cuda")
grid = gg.GGrid(g, cfg["cell_size"], max_objects=n_obj, log_capacity=1 << 27, async_ingest=True)
if len(pre):
    grid.ingest(torch.from_numpy(pre.view(np.int32)).cuda())
    grid.flush_all()
for h in hus + hqs:  # first DMA of each pinned buffer, untimed
    h.cuda()
torch.cuda.synchronize()


def loop(outs, steps, copy_back=False):
    grid.ingest_stage(hus[0])
    grid.query_stage(hqs[0])
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for s in range(steps):
        grid.ingest_commit()
        if s + 1 < steps:
            grid.ingest_stage(hus[s + 1])
            grid.query_stage(hqs[s + 1])
        grid.knn_commit(k, *outs)
        if copy_back:
            ho.copy_(outs[0], non_blocking=True)
            hd.copy_(outs[1], non_blocking=True)
            torch.cuda.current_stream().synchronize()
    grid.sync()
    return 1e3 * (time.perf_counter() - t0) / steps


def serial(steps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for s in range(steps):
        grid.ingest(hus[s])
        grid.knn(hqs[s], k, ho, hd)
    grid.sync()
    return 1e3 * (time.perf_counter() - t0) / steps


loop((ho, hd), 3)
res = {}
for rep in range(2):
    res.setdefault("inplace", []).append(loop((ho, hd), args.steps))
    res.setdefault("devout", []).append(loop((do, dd), args.steps, copy_back=True))
    res.setdefault("serial", []).append(serial(args.steps))
for n, v in res.items():
    print(f"{n:8s} ms/step {min(v):.3f}  ({Q / (min(v) / 1e3) / 1e6:.2f} M q/s)  all {[round(x, 3) for x in v]}")

if args.trace:
    from torch.profiler import ProfilerActivity, profile

    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        loop((ho, hd), 3)
    evs = sorted((e.time_range.start, e.time_range.end, e.name[:70]) for e in prof.events())
    with open(args.trace, "w") as f:
        for a, b, n in evs:
            f.write(f"{a - evs[0][0]:10.1f} {b - evs[0][0]:10.1f} {b - a:8.1f}  {n}\n")
    print("trace ->", args.trace)
grid.close()
