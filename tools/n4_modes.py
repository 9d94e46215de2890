"""N4: eager vs lazy message cleaning across the update frequency f, and the
single-query response time ("G-Grid (L)", P@61891-62321) next to the amortised batch time.

Workload: C1 (NY-shaped graph, |O| = 1e4, k = 10).  One time unit = f walk ticks (every object
reports f times, P@58136 "f = 1 update per second") followed by the unit's queries.
  lazy   : ingest(f ticks) ; knn(Q)                  (the paper's method, P@17773-17981)
  eager  : ingest(f ticks) ; flush_all ; knn(Q)      (every cell cleaned at update time)
Per mode and f: device time per unit (CUDA events on the library's stream) split by kernel
(profile mode), amortised time per query (T_u + T_q)/n_q (P@58274).
Latency: after each unit's ingest, L single-query ggrid_knn calls, each timed on the device and
on the host clock; mean = G-Grid (L).

Usage: python tools/n4_modes.py [--f 1,2,4,8,16,32,64] [--queries 10000] [--latency 64]
       [--out profiles/n4_modes_r01.jsonl]
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


def run(g, f, mode, Q, k, L, steps, warm, n_obj, cell_size, l2):
    walk = synth.RandomWalk(g, n_obj)
    stream = torch.cuda.Stream()
    grid = gg.GGrid(g, cell_size, max_objects=n_obj, profile=True, stream=stream.cuda_stream)
    out_o = torch.empty((Q, k), dtype=torch.int32, device="cuda")
    out_d = torch.empty_like(out_o)
    o1 = torch.empty((1, k), dtype=torch.int32, device="cuda")
    d1 = torch.empty_like(o1)
    grid.ingest(walk.tick())
    # single-query response times on an index without profile-mode events (each event pair
    # around a launch adds microseconds), fed the same update stream
    lwalk = synth.RandomWalk(g, n_obj)
    lgrid = gg.GGrid(g, cell_size, max_objects=n_obj, stream=stream.cuda_stream)
    lgrid.ingest(lwalk.tick())
    rows, lat_dev, lat_host = [], [], []
    for s in range(warm + steps):
        u = torch.from_numpy(walk.ticks(f).view(np.int32)).cuda()
        q = torch.from_numpy(synth.queries(g, Q, seed=synth.SEED_QUERIES + s).view(np.int32)).cuda()
        with torch.cuda.stream(stream):
            l2.zero_()
        torch.cuda.synchronize()
        grid.stats_reset()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        e[0].record(stream)
        grid.ingest(u)
        e[1].record(stream)
        if mode == "eager":
            grid.flush_all()
        e[2].record(stream)
        grid.knn(q, k, out_o, out_d)
        e[3].record(stream)
        torch.cuda.synchronize()
        km = grid.stats()["kernel_ms"]
        if s >= warm:
            rows.append(dict(unit_ms=e[0].elapsed_time(e[3]), ingest_ms=e[0].elapsed_time(e[1]),
                             eager_flush_ms=e[1].elapsed_time(e[2]), knn_ms=e[2].elapsed_time(e[3]),
                             k_flush_ms=km["flush"], k_expand_ms=km["expand"] + km["expand_big"]))
        # single-query response times after a fresh ingest (cells dirty again)
        if L and s >= warm:
            lgrid.ingest(torch.from_numpy(lwalk.ticks(f).view(np.int32)).cuda())
            if mode == "eager":
                lgrid.flush_all()
            q1 = torch.from_numpy(synth.queries(g, L, seed=99_000 + s).view(np.int32)).cuda()
            for i in range(L):
                a = torch.cuda.Event(enable_timing=True)
                b = torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                a.record(stream)
                lgrid.knn(q1[i:i + 1], k, o1, d1)
                b.record(stream)
                b.synchronize()
                lat_host.append(time.perf_counter() - t0)
                lat_dev.append(a.elapsed_time(b))
    grid.close()
    lgrid.close()
    med = {key: float(np.median([r[key] for r in rows])) for key in rows[0]}
    res = dict(mode=mode, f=f, objects=n_obj, Q=Q, k=k, updates_per_unit=f * n_obj, steps=steps, **med)
    res["amortised_us_per_query"] = 1e3 * med["unit_ms"] / Q
    res["qps"] = Q / (med["unit_ms"] / 1e3)
    if L:
        res["latency_dev_us_mean"] = 1e3 * float(np.mean(lat_dev))
        res["latency_host_us_mean"] = 1e6 * float(np.mean(lat_host))
        res["latency_host_us_p99"] = 1e6 * float(np.percentile(lat_host, 99))
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--f", default="1,2,4,8,16,32,64")
    ap.add_argument("--queries", type=int, default=10_000)
    ap.add_argument("--latency", type=int, default=64)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--objects", type=int, default=10_000)
    ap.add_argument("--k", type=int, default=10)
    ap.add_argument("--cell-size", type=int, default=1024)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "n4_modes_r01.jsonl"))
    a = ap.parse_args()
    g = synth.config_graph("C1")
    l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    with open(a.out, "w") as fo:
        for f in [int(x) for x in a.f.split(",")]:
            for mode in ("lazy", "eager"):
                r = run(g, f, mode, a.queries, a.k, a.latency, a.steps, a.warmup, a.objects, a.cell_size, l2)
                fo.write(json.dumps(r) + "\n")
                fo.flush()
                lat = (f"  Q=1 latency {r['latency_dev_us_mean']:7.1f} us dev / {r['latency_host_us_mean']:7.1f} us host"
                       if a.latency else "")
                print(f"f={f:>3} {mode:5s}: unit {r['unit_ms']:7.3f} ms = ingest {r['ingest_ms']:6.3f} + eager "
                      f"{r['eager_flush_ms']:6.3f} + knn {r['knn_ms']:6.3f}  -> {r['amortised_us_per_query']:6.3f} us/query "
                      f"({r['qps']/1e6:6.2f} Mq/s){lat}", flush=True)


if __name__ == "__main__":
    main()
