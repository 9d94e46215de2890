"""Does a staged H2D copy overlap the library's kernels?  Host wall times, C1 workload."""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402


def med(fn, reps=7):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    return 1e3 * float(np.median(ts))


side = torch.cuda.Stream()
src = torch.empty(16 << 20, dtype=torch.uint8).pin_memory()
dst = torch.empty(16 << 20, dtype=torch.uint8, device="cuda")
print(f"A copy alone                      {med(lambda: dst.copy_(src, non_blocking=True)):.3f} ms")
print(f"A sleep alone                     {med(lambda: torch.cuda._sleep(400_000)):.3f} ms")
def a_both():
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    torch.cuda._sleep(400_000)
print(f"A copy(side) + sleep(main)        {med(a_both):.3f} ms")

g = synth.config_graph("C1")
walk = synth.RandomWalk(g, 10_000)
grid = gg.GGrid(g, 1024, max_objects=10_000)
us = [torch.from_numpy(walk.ticks(100).view(np.int32)).pin_memory() for _ in range(4)]
dq = torch.from_numpy(synth.queries(g, 10_000).view(np.int32)).cuda()
do = torch.empty((10_000, 10), dtype=torch.int32, device="cuda")
dd = torch.empty_like(do)
grid.ingest(us[0])
grid.knn(dq, 10, do, dd)
print(f"B knn alone (device)              {med(lambda: grid.knn(dq, 10, do, dd)):.3f} ms")
def b_both():
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    grid.knn(dq, 10, do, dd)
print(f"B torch copy(side) + knn          {med(b_both):.3f} ms")
def c_both():
    grid.ingest_stage(us[1])
    torch.cuda._sleep(400_000)
    torch.cuda.synchronize()
    grid.ingest_commit()
def c_commit_only():
    grid.ingest_stage(us[1])
    torch.cuda.synchronize()
    grid.ingest_commit()
print(f"C stage+commit                    {med(c_commit_only):.3f} ms")
print(f"C stage + sleep(main) + commit    {med(c_both):.3f} ms")
def d_both():
    grid.ingest_stage(us[1])
    grid.knn(dq, 10, do, dd)
    torch.cuda.synchronize()
    grid.ingest_commit()
print(f"D stage + knn + commit            {med(d_both):.3f} ms")
# host-side timeline of D
torch.cuda.synchronize()
t0 = time.perf_counter()
grid.ingest_stage(us[2])
t1 = time.perf_counter()
grid.knn(dq, 10, do, dd)
t2 = time.perf_counter()
torch.cuda.synchronize()
t3 = time.perf_counter()
grid.ingest_commit()
t4 = time.perf_counter()
print(f"D timeline: stage {1e3*(t1-t0):.3f}  knn {1e3*(t2-t1):.3f}  drain {1e3*(t3-t2):.3f}  commit {1e3*(t4-t3):.3f} ms")
# the same with the library's stats (per-round syncs)
s0 = grid.stats()
grid.knn(dq, 10, do, dd)
s1 = grid.stats()
print("knn rounds per call", s1["knn_rounds"] - s0["knn_rounds"], "launches", s1["launches"] - s0["launches"])
# E: the bench's order (commit, stage next, knn)
grid.ingest_stage(us[1])
torch.cuda.synchronize()
k = [2]
def e_step():
    grid.ingest_commit()
    grid.ingest_stage(us[k[0]])
    k[0] = 1 + (k[0] % 3)
    grid.knn(dq, 10, do, dd)
print(f"E commit + stage + knn            {med(e_step):.3f} ms")
def e_nocopy():
    grid.ingest(dst_u)
    grid.knn(dq, 10, do, dd)
grid.ingest_commit()
dst_u = us[1].cuda()
print(f"E' ingest(device) + knn           {med(e_nocopy):.3f} ms")
grid.ingest_stage(us[1])
torch.cuda.synchronize()
for rep in range(3):
    t0 = time.perf_counter()
    grid.ingest_commit()
    t1 = time.perf_counter()
    grid.ingest_stage(us[1 + rep])
    t2 = time.perf_counter()
    grid.knn(dq, 10, do, dd)
    t3 = time.perf_counter()
    torch.cuda.synchronize()
    t4 = time.perf_counter()
    print(f"E timeline: commit {1e3*(t1-t0):.3f}  stage {1e3*(t2-t1):.3f}  knn {1e3*(t3-t2):.3f}  drain {1e3*(t4-t3):.3f} ms")
grid.ingest_commit()
# F: same with ingest of a staged batch but no copy in flight during knn
grid.ingest_stage(us[1])
def f_step():
    grid.ingest_commit()
    grid.knn(dq, 10, do, dd)
    grid.ingest_stage(us[1])
print(f"F commit + knn + stage(drained)   {med(f_step):.3f} ms")
grid.ingest_commit()
