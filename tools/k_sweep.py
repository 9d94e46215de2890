"""C2 k sweep (BASELINE configs[2]; the paper's Fig. 7 "varying k" analog, P@63498): FLA-shaped
graph, 1e5 objects, 10 cached updates per object per step, Q = 1e4 queries, k in {10..50}
(and beyond, up to the library's max_k).  Per k: device time per step (ingest + knn incl. lazy
flush), queries/s, expansion work per query, and a sampled bit-exact check against the oracle.

Usage: python tools/k_sweep.py [--k 10,20,30,40,50,100,200] [--out profiles/k_sweep_C2_r01.jsonl]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402  (parity sample only)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--k", default="10,20,30,40,50,100,200")
    ap.add_argument("--queries", type=int, default=10_000)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--parity", type=int, default=64)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "k_sweep_C2_r01.jsonl"))
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    g = synth.config_graph(a.config)
    l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    Q = a.queries
    with open(a.out, "w") as f:
        for k in [int(x) for x in a.k.split(",")]:
            walk = synth.RandomWalk(g, cfg["n_objects"])
            stream = torch.cuda.Stream()
            grid = gg.GGrid(g, cfg["cell_size"], max_objects=cfg["n_objects"], profile=True,
                            stream=stream.cuda_stream)
            oo = torch.empty((Q, k), dtype=torch.int32, device="cuda")
            od = torch.empty_like(oo)
            times, hist = [], []
            for s in range(a.warmup + a.steps):
                u = walk.ticks(cfg["updates_per_object"])
                hist.append(u)
                du = torch.from_numpy(u.view(np.int32)).cuda()
                qn = synth.queries(g, Q, seed=synth.SEED_QUERIES + s)
                dq = torch.from_numpy(qn.view(np.int32)).cuda()
                with torch.cuda.stream(stream):
                    l2.zero_()
                torch.cuda.synchronize()
                if s == a.warmup:
                    grid.stats_reset()
                    st0 = grid.stats()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                grid.ingest(du)
                grid.knn(dq, k, oo, od)
                e1.record(stream)
                e1.synchronize()
                if s >= a.warmup:
                    times.append(e0.elapsed_time(e1))
            st1 = grid.stats()
            sel = np.random.default_rng(k).choice(Q, a.parity, replace=False)
            ro, rd = oracle.knn_from_updates(g, np.concatenate(hist), qn[sel], k, mode=oracle.EARLY)
            go = oo.cpu().numpy().view(np.uint32)[sel]
            gd = od.cpu().numpy().view(np.uint32)[sel]
            exact = bool(np.array_equal(go, ro) and np.array_equal(gd, rd))
            n = Q * a.steps
            w = {x: (st1[f"expand_{x}"] - st0[f"expand_{x}"]) / n for x in ("iterations", "vertices", "arcs", "objects")}
            km = st1["kernel_ms"]
            r = dict(config=a.config, k=k, Q=Q, objects=cfg["n_objects"], ms_per_step=float(np.median(times)),
                     qps=Q / (float(np.median(times)) / 1e3), expand_ms=(km["expand"] + km["expand_big"]) / a.steps,
                     flush_ms=km["flush"] / a.steps, work_per_query=w, knn_rounds=(st1["knn_rounds"] - st0["knn_rounds"]) / a.steps,
                     parity_sample=a.parity, parity_exact=exact)
            f.write(json.dumps(r) + "\n")
            f.flush()
            print(f"{a.config} k={k:>4}: {r['qps']/1e6:6.2f} Mq/s  step {r['ms_per_step']:.3f} ms  expand {r['expand_ms']:.3f} ms  "
                  f"vertices/q {w['vertices']:.0f}  rounds {r['knn_rounds']:.1f}  parity({a.parity}) {exact}", flush=True)
            grid.close()


if __name__ == "__main__":
    main()
