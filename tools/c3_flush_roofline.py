"""USA-scale (BASELINE configs[3]) flush roofline + query batch + sampled parity.

  python tools/c3_flush_roofline.py [--ticks 64] [--queries 65536] [--parity 32]

1. USA-shaped graph (23,974,347 V / 58,333,344 arcs), 1M objects, `ticks` x 1M cached updates
   (64M records ~ 1.5 GB of SoA log, >> 126 MB L2) ingested in batches of 8M.
2. ggrid_flush_all once: flush-kernel CUDA-event time, algorithmic bytes,
   GB/s and fraction of the measured HBM peak.
3. one knn batch of `queries` (k=10) on the cleaned index: queries/s.
4. `parity` sampled queries checked bit-exact against the oracle (EARLY mode; 4 in FULL mode).
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
    ap.add_argument("--ticks", type=int, default=64)
    ap.add_argument("--objects", type=int, default=1_000_000)
    ap.add_argument("--queries", type=int, default=65536)
    ap.add_argument("--parity", type=int, default=32)
    ap.add_argument("--cell-size", type=int, default=1024)
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--batch-ticks", type=int, default=64, help="ticks per ingest call (extents per cell)")
    ap.add_argument("--repeat", type=int, default=4, help="ingest+flush rounds (median reported)")
    args = ap.parse_args()

    import torch

    import paper_conf_icde_li0qhdy18_b200 as gg
    import synth

    t0 = time.time()
    g = synth.table_ii_graph("USA", scale=args.scale)
    t_graph = time.time() - t0
    stream = torch.cuda.Stream()
    t0 = time.time()
    grid = gg.GGrid(g, args.cell_size, max_objects=args.objects, profile=True,
                    log_capacity=(args.objects * args.ticks + (8 << 20)) * (args.repeat + 1),
                    stream=stream.cuda_stream)
    t_build = time.time() - t0
    walk = synth.RandomWalk(g, args.objects)
    hist = []
    dev_batches = []
    for b in range(0, args.ticks, args.batch_ticks):
        u = walk.ticks(min(args.batch_ticks, args.ticks - b))
        if args.parity:
            hist.append(u)
        dev_batches.append(torch.from_numpy(u.view(np.int32)).cuda())
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    # Rounds: ingest the batches (the same messages again in later rounds: newer seq, same
    # locations), then one timed eager flush of every cell.  Reported: best and median round.
    rounds = []
    n_upd = 0
    for r in range(args.repeat):
        torch.cuda.synchronize()
        grid.stats_reset()
        for du in dev_batches:
            grid.ingest(du)
        st = grid.stats()
        ing_ms = sum(st["kernel_ms"][k] for k in ("ingest_classify", "ingest_alloc", "ingest_scatter"))
        n_upd = sum(len(d) for d in dev_batches)
        l2.zero_()
        torch.cuda.synchronize()
        s0 = grid.stats()
        grid.stats_reset()
        grid.flush_all()
        s1 = grid.stats()
        rec = s1["records_flushed"] - s0["records_flushed"]
        win = s1["objects_written"] - s0["objects_written"]
        cells = s1["cells_flushed"] - s0["cells_flushed"]
        alg = rec * 12 + win * 56  # DESIGN.md §4 (bench.py FLUSH_BYTES_*)
        rounds.append(dict(ingest_ms=ing_ms, flush_ms=s1["kernel_ms"]["flush"], rec=rec, win=win, cells=cells,
                           alg=alg, gc=s1["gc_runs"]))
    best = min(rounds, key=lambda x: x["flush_ms"])
    fl_ms = float(np.median([x["flush_ms"] for x in rounds]))
    ingest_ms = float(np.median([x["ingest_ms"] for x in rounds]))
    rec, win, cells, alg = best["rec"], best["win"], best["cells"], best["alg"]
    fl_gbs = alg / (fl_ms / 1e3) / 1e9
    # --- query batch
    q = synth.queries(g, args.queries)
    dq = torch.from_numpy(q.view(np.int32)).cuda()
    oo = torch.empty((args.queries, 10), dtype=torch.int32, device="cuda")
    od = torch.empty((args.queries, 10), dtype=torch.int32, device="cuda")
    grid.knn(dq, 10, oo, od)  # warm-up (also sizes the scratch buffers)
    torch.cuda.synchronize()
    grid.stats_reset()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    grid.knn(dq, 10, oo, od)
    e1.record(stream)
    e1.synchronize()
    knn_ms = e0.elapsed_time(e1)
    s2 = grid.stats()
    out = dict(config="C3 USA-shaped", n_vertices=int(g["n_vertices"]), n_arcs=int(len(g["src"])),
               objects=args.objects, cached_updates=n_upd, cell_size=s1["cell_size"], n_cells=s1["n_cells"],
               t_graph_s=t_graph, t_build_s=t_build,
               ingest_ms=ingest_ms, ingest_updates_per_s=n_upd / (ingest_ms / 1e3),
               ingest_gbs=n_upd * 48 / (ingest_ms / 1e3) / 1e9,
               flush_ms=fl_ms, flush_records=rec, flush_objects=win, flush_cells=cells, flush_alg_bytes=alg,
               flush_gbs=fl_gbs, flush_frac_of_peak=fl_gbs / peak, peak_gbs=peak,
               flush_best_gbs=best["alg"] / (best["flush_ms"] / 1e3) / 1e9,
               rounds=[{k: round(v, 4) if isinstance(v, float) else v for k, v in x.items()} for x in rounds],
               knn_queries=args.queries, knn_ms=knn_ms, knn_qps=args.queries / (knn_ms / 1e3),
               knn_kernel_ms=s2["kernel_ms"], knn_rounds=s2["knn_rounds"])
    # --- sampled parity
    if args.parity:
        import oracle

        ids, e, d = oracle.snapshot_objects(np.concatenate(hist), args.objects)
        sel = np.linspace(0, args.queries - 1, args.parity).astype(np.int64)
        t0 = time.time()
        ro, rd = oracle.knn(g, ids, e, d, q[sel], 10, mode=oracle.EARLY)
        go = oo.cpu().numpy().view(np.uint32)[sel]
        gd = od.cpu().numpy().view(np.uint32)[sel]
        out["parity_early_ok"] = bool(np.array_equal(go, ro) and np.array_equal(gd, rd))
        out["parity_early_n"] = int(len(sel))
        ro4, rd4 = oracle.knn(g, ids, e, d, q[sel[:4]], 10, mode=oracle.FULL)
        out["parity_full_ok"] = bool(np.array_equal(go[:4], ro4) and np.array_equal(gd[:4], rd4))
        out["parity_s"] = time.time() - t0
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
