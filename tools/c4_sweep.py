"""C4 update-heavy sweep (the paper's Fig. 8/9 update-frequency analog).

For graph in {C1 (NY-shaped), C2 (FLA-shaped)}, |O| in {1e4, 1e5, 1e6} and r in {10 .. 1e5}
updates per query: each step ingests r*Q updates (device-resident, generated on the GPU by
synth.device_walk) and answers Q = 1e4 queries with k = 10.  The per-kernel CUDA-event
timings of profile mode split the step into ingest / flush / query (seed + expand), giving the
T_flush vs T_query crossover SURVEY §8(d) predicts near r ~ 750 (bytes).

Usage: python tools/c4_sweep.py [--graphs C1,C2] [--objects 1e4,1e5,1e6] [--r 10,...]
       [--out profiles/c4_sweep.jsonl]
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402
from synth.device_walk import DeviceRandomWalk  # noqa: E402

SEQ_LIMIT = (1 << 32) - 1
TRACE = os.environ.get("C4_TRACE")


def run_one(g, gname, n_obj, r, Q, k, cell_size, max_steps, l2):
    n_upd = int(r * Q)
    walk = DeviceRandomWalk(g, n_obj)
    ticks = -(-n_upd // n_obj)
    buf = torch.empty((ticks * n_obj, 4), dtype=torch.int32, device="cuda")
    n_steps = max(1, min(max_steps, (SEQ_LIMIT - n_obj) // n_upd - 1))
    cap = int(n_upd * 1.05) + 8 * n_obj + (1 << 22)
    grid = gg.GGrid(g, cell_size, max_objects=n_obj, profile=True, log_capacity=cap)
    out_o = torch.empty((Q, k), dtype=torch.int32, device="cuda")
    out_d = torch.empty_like(out_o)
    grid.ingest(walk.ticks(1))  # every object placed (ordered after the walk kernels: the binding
    # makes the library stream wait for torch's current stream, ggrid_wait_stream)
    rows = []
    gen_s = 0.0
    for s in range(1 + n_steps):  # step 0 = warm-up
        t0 = time.perf_counter()
        u = walk.ticks_into(buf, ticks)[:n_upd]
        q = torch.from_numpy(synth.queries(g, Q, seed=synth.SEED_QUERIES + s).view(np.int32)).cuda()
        torch.cuda.synchronize()
        gen_s += time.perf_counter() - t0
        l2.zero_()
        torch.cuda.synchronize()
        grid.stats_reset()
        st0 = grid.stats()
        prof = None
        if TRACE and s == n_steps:
            from torch.profiler import ProfilerActivity, profile
            prof = profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU])
            prof.__enter__()
        e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        e0.record()
        grid.ingest(u)
        e1.record()
        grid.knn(q, k, out_o, out_d)
        e2.record()
        torch.cuda.synchronize()
        if prof is not None:
            prof.__exit__(None, None, None)
            evs = sorted((e.time_range.start, e.time_range.end, e.name[:70]) for e in prof.events())
            with open(TRACE, "w") as f:
                for a, b, nm in evs:
                    f.write(f"{a - evs[0][0]:10.1f} {b - evs[0][0]:10.1f} {b - a:8.1f}  {nm}\n")
        st = grid.stats()
        for key in ("records_flushed", "cells_flushed", "objects_written", "knn_rounds", "gc_runs"):
            st[key] -= st0[key]
        if s == 0:
            continue
        km = st["kernel_ms"]
        ing = km["ingest_classify"] + km["ingest_alloc"] + km["ingest_scatter"]
        rows.append(dict(step_ms=e0.elapsed_time(e2), ingest_call_ms=e0.elapsed_time(e1),
                         knn_call_ms=e1.elapsed_time(e2), ingest_ms=ing, flush_ms=km["flush"],
                         seed_ms=km["seed"], expand_ms=km["expand"] + km["expand_big"],
                         other_ms=km["other"], records_flushed=st["records_flushed"],
                         cells_flushed=st["cells_flushed"], objects_written=st["objects_written"],
                         knn_rounds=st["knn_rounds"], gc_runs=st["gc_runs"]))
    grid.close()
    del buf
    torch.cuda.empty_cache()
    med = {key: float(np.median([row[key] for row in rows])) for key in rows[0]}
    return dict(graph=gname, n_vertices=g["n_vertices"], objects=n_obj, r=r, Q=Q, k=k,
                cell_size=cell_size, updates_per_step=n_upd, steps=len(rows),
                qps=Q / (med["step_ms"] / 1e3), updates_per_s=n_upd / (med["ingest_ms"] / 1e3),
                flush_gbs=(12 * med["records_flushed"] + 56 * med["objects_written"]) / (med["flush_ms"] / 1e3) / 1e9
                if med["flush_ms"] > 0 else None,
                ingest_gbs=48 * n_upd / (med["ingest_ms"] / 1e3) / 1e9, gen_s=gen_s, **med)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graphs", default="C1,C2")
    ap.add_argument("--objects", default="1e4,1e5,1e6")
    ap.add_argument("--r", default="10,100,1000,10000,100000")
    ap.add_argument("--queries", type=int, default=10_000)
    ap.add_argument("--k", type=int, default=10)
    ap.add_argument("--cell-size", type=int, default=1024)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--max-updates", type=float, default=1.0e9, help="skip combos above this")
    ap.add_argument("--max-ticks", type=float, default=2.0e4,
                    help="skip combos whose step needs more walk ticks (generator time)")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "c4_sweep.jsonl"))
    a = ap.parse_args()
    l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    with open(a.out, "w") as f:
        for cfg in a.graphs.split(","):
            g = synth.config_graph(cfg)
            for n_obj in [int(float(x)) for x in a.objects.split(",")]:
                for r in [int(float(x)) for x in a.r.split(",")]:
                    if r * a.queries > a.max_updates or r * a.queries / n_obj > a.max_ticks:
                        print(f"{cfg} |O|={n_obj:>8} r={r:>6}: skipped (generator budget)", flush=True)
                        continue
                    res = run_one(g, cfg, n_obj, r, a.queries, a.k, a.cell_size, a.steps, l2)
                    f.write(json.dumps(res) + "\n")
                    f.flush()
                    print(f"{cfg} |O|={n_obj:>8} r={r:>6}: {res['qps']/1e6:7.3f} Mq/s  step {res['step_ms']:9.3f} ms "
                          f"= ingest {res['ingest_ms']:8.3f} + flush {res['flush_ms']:8.3f} + seed {res['seed_ms']:6.3f} "
                          f"+ expand {res['expand_ms']:7.3f}  flush {res['flush_gbs'] or 0:7.1f} GB/s  "
                          f"ingest {res['ingest_gbs']:7.1f} GB/s  gen {res['gen_s']:.1f}s", flush=True)


if __name__ == "__main__":
    main()
