"""N3: the paper's query pipeline -- GPU candidate cells + Bellman-Ford + first-k +
unresolved vertices (Alg. 4-5, Def. 3), then Refine_kNN on CPU threads (Alg. 6) -- timed beside
the fused GPU expansion (ggrid_knn) on the same index and the same queries; both checked equal,
and a sample checked against the oracle.

    python tools/n3_refine.py [--config C1|C3] [--queries 2048] [--rho 1.8] [--threads 0]
Prints one JSON line.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C1")
    ap.add_argument("--queries", type=int, default=2048)
    ap.add_argument("--rho", type=float, default=1.8)
    ap.add_argument("--threads", type=int, default=0)
    ap.add_argument("--parity", type=int, default=64)
    args = ap.parse_args()
    import torch

    import oracle
    import paper_conf_icde_li0qhdy18_b200 as gg
    import synth

    cfg = dict(synth.CONFIGS[args.config])
    cfg.update(synth.BENCH_STEPS[args.config])
    g = synth.config_graph(args.config)
    walk = synth.RandomWalk(g, cfg["n_objects"])
    upd = walk.ticks(max(cfg["preload_ticks"], cfg["step_ticks"]))
    grid = gg.GGrid(g, cfg["cell_size"], max_objects=cfg["n_objects"], log_capacity=1 << 27)
    grid.ingest(torch.from_numpy(upd.view(np.int32)).cuda())
    grid.flush_all()
    q = synth.queries(g, args.queries, seed=77)
    k = cfg["k"]
    grid.knn(q, k)  # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    go, gd = grid.knn(q, k)
    t_fused = time.perf_counter() - t0
    grid.prior_art_knn(q[:64], k, rho=args.rho, threads=args.threads)  # warm-up (host CSR copy)
    t0 = time.perf_counter()
    po, pd, res = grid.prior_art_knn(q, k, rho=args.rho, threads=args.threads)
    t_pa = time.perf_counter() - t0
    same = bool(np.array_equal(go, po) and np.array_equal(gd, pd))
    sel = np.linspace(0, len(q) - 1, min(args.parity, len(q))).astype(np.int64)
    ids, e, d = oracle.snapshot_objects(upd, cfg["n_objects"])
    ro, rd = oracle.knn(g, ids, e, d, q[sel], k, mode=oracle.EARLY)
    exact = bool(np.array_equal(go[sel], ro) and np.array_equal(gd[sel], rd))
    nq = len(q)
    query_ms = res["ms_gpu"] + res["ms_d2h"] + res["ms_cpu_refine"]
    out = dict(config=args.config, queries=nq, k=k, rho=args.rho,
               fused_gpu={"wall_ms": 1e3 * t_fused, "qps": nq / t_fused},
               prior_art={"wall_ms": 1e3 * t_pa, "query_ms": query_ms, "qps_query_phase": nq / (query_ms / 1e3),
                          **{kk: (v / nq if kk in ("cells", "vertices", "bf_iterations", "unresolved", "refine_settled")
                                  else v) for kk, v in res.items()}},
               per_query_note="cells/vertices/bf_iterations/unresolved/refine_settled are per-query means",
               speedup_fused_over_prior_art=(query_ms / 1e3) / t_fused, answers_equal=same,
               oracle_rows=int(len(sel)), oracle_exact=exact)
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
