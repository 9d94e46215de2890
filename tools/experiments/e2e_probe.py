"""Where does the end-to-end step (host buffers) spend its time?  C1 workload.

Times (wall clock, after warm-up): plain H2D copy of one update batch; ggrid_ingest from
pinned host; ggrid_knn with pinned host queries/answers; the pipelined stage/commit loop.
"""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402


def wall(fn, reps=5):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    return 1e3 * float(np.median(ts))


g = synth.config_graph("C1")
walk = synth.RandomWalk(g, 10_000)
grid = gg.GGrid(g, 1024, max_objects=10_000)
us = [torch.from_numpy(walk.ticks(100).view(np.int32)).pin_memory() for _ in range(12)]
q = torch.from_numpy(synth.queries(g, 10_000).view(np.int32)).pin_memory()
ho = torch.empty((10_000, 10), dtype=torch.int32).pin_memory()
hd = torch.empty((10_000, 10), dtype=torch.int32).pin_memory()
dev = torch.empty_like(us[0], device="cuda")
grid.ingest(us[0])
grid.knn(q, 10, ho, hd)
print(f"H2D 16 MB pinned copy            {wall(lambda: dev.copy_(us[1], non_blocking=True)):.3f} ms")
it = iter(us[1:])
print(f"ggrid_ingest (pinned host)       {wall(lambda: grid.ingest(next(it)), 3):.3f} ms")
print(f"ggrid_ingest (device)            {wall(lambda: grid.ingest(dev), 3):.3f} ms")
print(f"ggrid_knn (pinned q/out)         {wall(lambda: grid.knn(q, 10, ho, hd)):.3f} ms")
dq = q.cuda()
do = torch.empty((10_000, 10), dtype=torch.int32, device="cuda")
dd = torch.empty_like(do)
print(f"ggrid_knn (device q/out)         {wall(lambda: grid.knn(dq, 10, do, dd)):.3f} ms")
# fresh cells to flush: ingest then knn, both paths
def step_dev():
    grid.ingest(dev)
    grid.knn(dq, 10, do, dd)
print(f"step device (ingest+knn)         {wall(step_dev, 3):.3f} ms")
it2 = iter(us[4:])
def step_host():
    grid.ingest(next(it2))
    grid.knn(q, 10, ho, hd)
print(f"step host (ingest+knn)           {wall(step_host, 3):.3f} ms")
it3 = iter(us[7:])
grid.ingest_stage(next(it3))
def step_pipe():
    grid.ingest_commit()
    grid.ingest_stage(next(it3))
    grid.knn(q, 10, ho, hd)
print(f"step pipelined (commit,stage,knn) {wall(step_pipe, 3):.3f} ms")
grid.ingest_commit()
# isolate: pipelined loop with device-resident queries/answers (only the staging copy on PCIe)
us2 = [torch.from_numpy(walk.ticks(100).view(np.int32)).pin_memory() for _ in range(6)]
it4 = iter(us2)
grid.ingest_stage(next(it4))
def step_pipe_dev():
    grid.ingest_commit()
    grid.ingest_stage(next(it4))
    grid.knn(dq, 10, do, dd)
print(f"step pipelined, device q/out      {wall(step_pipe_dev, 3):.3f} ms")
grid.ingest_commit()
# host-side cost of the stage call and of a commit whose copy finished long ago
grid.ingest_stage(us2[0])
torch.cuda.synchronize()
time.sleep(0.01)
t0 = time.perf_counter(); grid.ingest_commit(); t1 = time.perf_counter()
print(f"commit of an already-copied batch {1e3*(t1-t0):.3f} ms")
t0 = time.perf_counter(); grid.ingest_stage(us2[1]); t1 = time.perf_counter()
print(f"stage call (host time)            {1e3*(t1-t0):.3f} ms")
torch.cuda.synchronize()
grid.ingest_commit()
