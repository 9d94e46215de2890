"""Benchmark: kNN queries/s including the lazy flush at a fixed update rate (BASELINE.json).

One step = one pass of the whole hot path over one batch of synthetic input:
  ggrid_ingest(r*Q cached location updates)   (Alg. 1: a0)
  ggrid_knn(Q queries, k)                      (cell selection, lazy flush, expansion,
                                                 candidate top-k, unresolved, refinement:
                                                 a1-a6 of SURVEY §8(a))
value = queries answered / device time of the steps (CUDA events on the library's stream,
max over ranks).  Default workload: BASELINE configs[1] (NY-shaped graph, 10k objects,
1M cached updates per step = 100 ticks of the random walk, Q = 10^4 queries, k = 10).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C1|C0|C2|C3]
    python bench.py --impl reference ...    # the CPU oracle as the reference arm
Multi-GPU (torchrun): each rank owns a replica of the index, ingests the same update
stream and answers its own Q queries (weak scaling of the query work).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

CONFIG_TEXT = {
    "C0": "Fig.1-scale toy: ~1k-vertex synthetic grid road graph, 100 moving objects, 1k cached updates, k=3, 100 queries",
    "C1": "NY-shaped synthetic road graph (~264k vertices, ~734k edges), 10k objects, k=10, 1M cached updates",
    "C2": "FLA-shaped synthetic road graph (~1.07M vertices), 100k objects, k=10-50 sweep",
    "C3": "USA-shaped synthetic road graph (~24M vertices, ~58M edges), 1M objects, k=10, batched queries",
}
METRIC = "kNN queries/sec incl. lazy flush at fixed update rate"

# Algorithmic bytes per unit (restated in DESIGN.md §5)
INGEST_BYTES_PER_UPDATE = 48          # 16 record + 4 arc->cell + 8 RED.MAX + 20 SoA write
FLUSH_BYTES_PER_RECORD = 12           # obj + key (ot_key match is an L1-resident gather)
FLUSH_BYTES_PER_WINNER = 12 + 24 + 8 + 12  # payload read + compacted write + v_obj set + (next flush) clear
# expansion: counted work (ggrid_stats expand_*), bytes each unit must move
EXPAND_BYTES_PER_VERTEX = 8    # rowptr[u], rowptr[u+1]
EXPAND_BYTES_PER_ARC = 8       # adj (dst, w)
EXPAND_BYTES_PER_HARVEST = 12  # cell_head (dirty check) + v_obj (start, count)
EXPAND_BYTES_PER_OBJECT = 28   # obj, key, edge, off + ot_key (validity)
EXPAND_BYTES_PER_QUERY = 16    # query (edge, off) + inverted index (src, w)

# opts.profile masks (include/ggrid.h): bit 0 = every launch kind, bit k+1 = kind k.  A timed
# launch costs ~3-4 us of device idle time per event, so the timed steps time only the
# dominant kernel (the expansion, GGRID_K_EXPAND = 5 / GGRID_K_EXPAND_BIG = 6); the
# per-kernel split comes from extra, untimed breakdown steps with every launch timed.
PROFILE_ALL = 1
PROFILE_EXPAND = (2 << 5) | (2 << 6)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def workload(cfg: str, queries: int | None):
    c = dict(synth.CONFIGS[cfg])
    if queries:
        c["n_queries"] = queries
    return c


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(gpu), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def _rows(self):
        return [r.split(",") for r in open(self.f.name).read().strip().splitlines() if r.strip()]

    def mark(self):
        """Start of the timed region: samples before it (warm-up) are kept only as a fallback."""
        self.mark_rows = len(self._rows()) if self.p is not None else 0

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = self._rows()
        os.unlink(self.f.name)
        window = "timed steps"
        timed = rows[getattr(self, "mark_rows", 0):]
        if timed:
            rows = timed
        else:  # a timed region shorter than the 100 ms sampling interval: the warm-up's last samples
            rows = rows[-3:]
            window = "last warm-up samples (timed region shorter than the sampling interval)"
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            r = [x.strip() for x in r]
            try:
                sm.append(float(r[1]))
                mx.append(float(r[2]))
            except (ValueError, IndexError):
                continue
            for n, v in zip(names, r[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm), "window": window}


def dist_setup():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


# -------------------------------------------------------------------------- oracle arm
def time_oracle(g, cfg, upd_step, queries, n_sample, threads=0):
    """The CPU oracle as it stands on a bounded sample: snapshot of one step's updates +
    n_sample full-Dijkstra queries; returns (queries/s scaled to the step, sample text, cores)."""
    import oracle

    cores = threads if threads > 0 else oracle.hardware_threads()
    snap = oracle.Snapshot(cfg["n_objects"])
    t0 = time.perf_counter()
    snap.apply(upd_step)
    t_snap = time.perf_counter() - t0
    ids, e, d = snap.objects()
    qs = queries[:n_sample]
    t0 = time.perf_counter()
    oracle.knn(g, ids, e, d, qs, cfg["k"], mode=oracle.FULL, threads=cores)
    t_q = time.perf_counter() - t0
    Q = len(queries)
    per_step = t_snap + t_q * Q / len(qs)
    sample = (f"snapshot of one step's {len(upd_step)} updates ({t_snap:.3f}s) + {len(qs)} of the step's {Q} "
              f"queries, full-graph Dijkstra ({t_q:.2f}s), scaled to the step")
    return Q / per_step, sample, cores


def run_reference(args, cfg_name):
    world, rank, _ = dist_setup()
    if world > 1 and rank != 0:
        return
    cfg = workload(cfg_name, args.queries)
    g = synth.config_graph(cfg_name)
    walk = synth.RandomWalk(g, cfg["n_objects"])
    n_sample = args.ref_sample
    times = []
    sample_txt, cores = "", 0
    for s in range(args.warmup + args.steps):
        upd = walk.ticks(cfg["updates_per_object"])
        q = synth.queries(g, cfg["n_queries"], seed=synth.SEED_QUERIES + s)
        qps, sample_txt, cores = time_oracle(g, cfg, upd, q, n_sample)
        if s >= args.warmup:
            times.append(cfg["n_queries"] / qps)
    value = cfg["n_queries"] * len(times) / sum(times)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic", "config": {"workload": CONFIG_TEXT[cfg_name], "config_id": cfg_name,
                                            "queries_per_step": cfg["n_queries"], "k": cfg["k"]},
            "cpu_baseline": {"value": value, "unit": "queries/s", "cores": cores, "kind": "oracle",
                             "sample": sample_txt},
            "e2e": {"value": value, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def run_ours(args, cfg_name):
    import torch

    import paper_conf_icde_li0qhdy18_b200 as gg

    world, rank, local = dist_setup()
    if world > 1:
        import torch.distributed as dist

        # one process per GPU over NCCL; BENCH_DIST_BACKEND=gloo lets the harness be exercised
        # with several ranks sharing one GPU (a test mode, not a measurement)
        backend = os.environ.get("BENCH_DIST_BACKEND", "nccl")
        dev_i = local % max(1, torch.cuda.device_count())
        torch.cuda.set_device(dev_i)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_i))
        else:
            dist.init_process_group(backend)
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()
    cfg = workload(cfg_name, args.queries)
    Q, k = cfg["n_queries"], cfg["k"]
    g = synth.config_graph(cfg_name)
    walk = synth.RandomWalk(g, cfg["n_objects"])
    stream = torch.cuda.Stream()
    shard = world > 1 and args.parallel == "shard"
    grid = gg.GGrid(g, args.cell_size or cfg["cell_size"], max_objects=cfg["n_objects"], profile=PROFILE_EXPAND,
                    log_capacity=args.log_capacity, delta=args.delta, stream=stream.cuda_stream,
                    async_ingest=True)
    if shard:  # cell-ownership sharding: logs of own cells only
        grid.shard(world, rank)
    out_o = torch.empty((Q, k), dtype=torch.int32, device="cuda")
    out_d = torch.empty((Q, k), dtype=torch.int32, device="cuda")
    # > 126 MB L2 (BENCH_L2_MB: diagnostics only, e.g. a longer flush lets the host run further ahead)
    l2 = torch.empty(int(os.environ.get("BENCH_L2_MB", "256")) << 20, dtype=torch.uint8, device="cuda")

    def step_inputs(s):
        u = walk.ticks(cfg["updates_per_object"])
        q = synth.queries(g, Q, seed=synth.SEED_QUERIES + 1000 * rank + s)
        return u, q

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()

    # ---- device-resident timed region -------------------------------------------------
    times = []
    st0 = None
    from paper_conf_icde_li0qhdy18_b200 import dist as gdist

    n_upd_step = cfg["n_objects"] * cfg["updates_per_object"]
    remote_requests = 0
    n_break = max(3, min(args.steps, 10))  # breakdown steps (every launch timed), after the timed ones
    for s in range(args.warmup + args.steps + n_break):
        q = synth.queries(g, Q, seed=synth.SEED_QUERIES + 1000 * rank + s)
        u = walk.ticks(cfg["updates_per_object"])  # every rank keeps the walk in step (untimed)
        if rank == 0:  # the update stream arrives at rank 0 and is fanned out over NCCL
            du = torch.from_numpy(u.view(np.int32)).to("cuda")
        else:
            du = torch.empty((n_upd_step, 4), dtype=torch.int32, device="cuda")
        dq = torch.from_numpy(q.view(np.int32)).to("cuda")
        barrier()
        if s == 0:  # (started with the warm-up: nvidia-smi needs ~0.1-0.3 s to report)
            clocks = ClockSampler(dev)
        if s == args.warmup:
            grid.stats_reset()
            st0 = grid.stats()
            clocks.mark()
        if s == args.warmup + args.steps:  # end of the timed steps
            clk = clocks.stop()
            grid.sync()  # (raises a deferred ingest error, if any)
            st1 = grid.stats()
            grid.set_profile(PROFILE_ALL)
            grid.stats_reset()
            sb0 = grid.stats()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            # flush L2 between timed iterations (outside the events); the host queues the
            # step's launches while the device is still writing it
            l2.zero_()
        e0.record(stream)
        if world > 1:
            with torch.cuda.stream(stream):
                gdist.broadcast_updates(du, src=0)
        grid.ingest(du)
        if shard:  # owner search + bounded requests/replies + merge, all ordered on `stream`
            with torch.cuda.stream(stream):
                out_o, out_d, n_req = gdist.sharded_knn(grid, dq, k, world, rank)
                remote_requests += n_req if args.warmup <= s < args.warmup + args.steps else 0
        else:
            grid.knn(dq, k, out_o, out_d)
        e1.record(stream)
        e1.synchronize()
        if args.warmup <= s < args.warmup + args.steps:
            times.append(e0.elapsed_time(e1))
    barrier()
    grid.sync()
    sb1 = grid.stats()
    total_ms = sum(times)
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device="cuda")
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        total_ms = float(t.item())
    K = args.steps
    value = world * Q * K / (total_ms / 1e3)
    n_upd = cfg["n_objects"] * cfg["updates_per_object"]

    # ---- per-kernel roofline ----------------------------------------------------------------
    # split: the breakdown steps (every launch timed); the dominant kernel's achieved rate: its
    # CUDA events inside the timed steps when it is the expansion (timed there), else the split
    peak, peak_kind = load_peaks()
    cs = st1["cell_size"]

    def kernels(a, b, nsteps):
        kms, kl = b["kernel_ms"], b["kernel_launches"]
        rec = b["records_flushed"] - a["records_flushed"]
        win = b["objects_written"] - a["objects_written"]
        dx = {n: b["expand_" + n] - a["expand_" + n] for n in ("iterations", "vertices", "arcs", "harvested", "objects")}
        expand_bytes = (dx["vertices"] * EXPAND_BYTES_PER_VERTEX + dx["arcs"] * EXPAND_BYTES_PER_ARC
                        + dx["harvested"] * EXPAND_BYTES_PER_HARVEST + dx["objects"] * EXPAND_BYTES_PER_OBJECT
                        + Q * nsteps * (EXPAND_BYTES_PER_QUERY + 8 * k))
        kern = {
            "ingest": (kms["ingest_classify"] + kms["ingest_alloc"] + kms["ingest_scatter"],
                       n_upd * nsteps * INGEST_BYTES_PER_UPDATE,
                       kl["ingest_classify"] + kl["ingest_alloc"] + kl["ingest_scatter"]),
            "flush": (kms["flush"], rec * FLUSH_BYTES_PER_RECORD + win * FLUSH_BYTES_PER_WINNER, kl["flush"]),
            # (level-0 launches: the chained level above runs beside them on a second stream,
            # so its event time overlaps theirs; its work is in the bytes)
            "expand": (kms["expand"], expand_bytes, kl["expand"]),
        }
        return kern, dx

    kern, _ = kernels(sb0, sb1, n_break)
    kern_t, dx = kernels(st0, st1, K)
    ingest_ms = kern["ingest"][0] * K / n_break  # ingest time of K steps, from the split
    dom = max(kern, key=lambda n: kern[n][0])
    dms, dbytes, dl = kern_t[dom] if dom == "expand" else kern[dom]
    achieved = dbytes / (dms / 1e3) / 1e9 if dms > 0 else 0.0
    per_kernel = {n: {"ms_per_step": v[0] / n_break, "launches_per_step": v[2] / n_break,
                      "alg_bytes_per_step": v[1] / n_break,
                      "gbs": (v[1] / (v[0] / 1e3) / 1e9) if v[0] > 0 else 0.0} for n, v in kern.items()}
    per_kernel["source"] = f"{n_break} breakdown steps after the timed ones, every launch timed"
    per_kernel["expand"]["level0_ms_per_step"] = sb1["kernel_ms"]["expand"] / n_break
    per_kernel["expand"]["higher_levels_ms_per_step"] = sb1["kernel_ms"]["expand_big"] / n_break
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"traffic_{cfg_name}.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp)).get(dom)
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": dom, "peak_source": peak_kind,
                "launch_ms": dms / max(1, dl), "timed_in": "timed steps" if dom == "expand" else "breakdown steps"}
    lp = os.path.join(ROOT, "profiles", f"limiters_{cfg_name}.json")
    if os.path.exists(lp):  # what bounds the kernel when it is not HBM (ncu, the last profiling pass)
        roofline["ncu_limiters"] = json.load(open(lp)).get(dom)
    updates_per_s = n_upd * K / (ingest_ms / 1e3) if ingest_ms > 0 else None

    # ---- e2e through the public API with pinned host buffers -------------------------------
    # Pipelined (ggrid_ingest_stage / ggrid_query_stage, then ggrid_ingest_commit /
    # ggrid_knn_commit, P@45017-45625): the next step's update and query batches are copied
    # from pinned host memory while this step's queries run.  The
    # timed region holds every step's H2D copies, the ingest, the queries and the D2H of the
    # answers; the warm-up step (s = 0) is excluded.
    # a fresh index without profile-mode events (a timing event queued behind a staged copy
    # costs ~50 us), warmed by the same stream of steps
    grid.close()
    grid = gg.GGrid(g, args.cell_size or cfg["cell_size"], max_objects=cfg["n_objects"],
                    log_capacity=args.log_capacity, delta=args.delta, async_ingest=True)
    if shard:
        grid.shard(world, rank)
    dq_e = torch.empty((Q, 2), dtype=torch.int32, device="cuda")

    def e2e_stage(hu, hq):
        grid.ingest_stage(hu)
        if not shard:
            grid.query_stage(hq)  # copied behind the update batch on the library's copy stream

    def e2e_knn(hq):
        if not shard:
            grid.knn_commit(k, h_o, h_d)  # the staged queries; answers written to pinned memory in place
            return
        dq_e.copy_(hq, non_blocking=True)
        o, d_, _ = gdist.sharded_knn(grid, dq_e, k, world, rank)
        h_o.copy_(o, non_blocking=True)
        h_d.copy_(d_, non_blocking=True)
        torch.cuda.current_stream().synchronize()
    h_o = torch.empty((Q, k), dtype=torch.int32).pin_memory()
    h_d = torch.empty((Q, k), dtype=torch.int32).pin_memory()
    n_e2e = max(1, args.e2e_steps)
    hus, hqs = [], []
    w_e2e = 3
    for s in range(w_e2e + n_e2e):
        u, q = step_inputs(10_000 + s)
        hus.append(torch.from_numpy(u.view(np.int32)).pin_memory())
        hqs.append(torch.from_numpy(q.view(np.int32)).pin_memory())
    # one untimed DMA from every pinned input buffer (a producer would reuse a fixed set of
    # pinned buffers; the first DMA from a freshly pinned allocation is measurably slower)
    scratch_u = torch.empty_like(hus[0], device="cuda")
    scratch_q = torch.empty_like(hqs[0], device="cuda")
    for hu, hq in zip(hus, hqs):
        scratch_u.copy_(hu)
        scratch_q.copy_(hq)
    torch.cuda.synchronize()
    del scratch_u, scratch_q
    for s in range(w_e2e):  # warm-up steps
        e2e_stage(hus[s], hqs[s])
        grid.ingest_commit()
        e2e_knn(hqs[s])
    hus, hqs = hus[w_e2e:], hqs[w_e2e:]
    hus.insert(0, None)
    hqs.insert(0, None)
    barrier()
    trace = None
    if os.environ.get("BENCH_E2E_TRACE"):  # diagnostics: CUPTI timeline of the e2e loop
        from torch.profiler import ProfilerActivity, profile
        trace = profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU])
        trace.__enter__()
    t0 = time.perf_counter()
    tst = []
    promo = []
    e2e_stage(hus[1], hqs[1])
    for s in range(1, n_e2e + 1):
        grid.ingest_commit()
        if s + 1 <= n_e2e:
            e2e_stage(hus[s + 1], hqs[s + 1])  # overlaps the queries below
        e2e_knn(hqs[s])
        tst.append(time.perf_counter())
        if os.environ.get("BENCH_E2E_DEBUG"):  # (perturbs the timing it reports)
            sd = grid.stats()
            promo.append((sd["expand_promotions"], sd["knn_rounds"]))
    if os.environ.get("BENCH_E2E_DEBUG"):
        print("e2e step ms:", [round(1e3 * (b - a), 3) for a, b in zip([t0] + tst[:-1], tst)], file=sys.stderr)
        print("e2e (promotions, knn rounds) after each step:", promo, file=sys.stderr)
        sd = grid.stats()
        print("e2e stats:", {k: sd[k] for k in ("gc_runs", "knn_rounds", "knn_calls", "expand_promotions",
                                                "expand_retries", "arena_used", "arena_capacity")}, file=sys.stderr)
    grid.sync()  # (the last step's answers were read back inside knn already)
    e2e_total = time.perf_counter() - t0
    if trace is not None:
        trace.__exit__(None, None, None)
        evs = sorted((e.time_range.start, e.time_range.end, e.name[:70]) for e in trace.events())
        with open(os.environ["BENCH_E2E_TRACE"], "w") as f:
            for a, b, n in evs:
                f.write(f"{a - evs[0][0]:10.1f} {b - evs[0][0]:10.1f} {b - a:8.1f}  {n}\n")
    e2e_times = [e2e_total / n_e2e] * n_e2e
    if world > 1:
        t = torch.tensor([e2e_total], dtype=torch.float64, device="cuda")
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        e2e_total = float(t.item())
    e2e = {"value": world * Q * len(e2e_times) / e2e_total, "unit": "queries/s",
           "h2d_bytes_per_step": n_upd * 16 + Q * 8, "d2h_bytes_per_step": Q * k * 8}

    # ---- CPU oracle beside it (rank 0, N=1 only) -------------------------------------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        u, q = step_inputs(20_000)
        qps, sample, cores = time_oracle(g, cfg, u, q, args.ref_sample)
        cpu = {"value": qps, "unit": "queries/s", "cores": cores, "kind": "oracle", "sample": sample}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": world, "steps": K,
                "warmup": args.warmup, "ms_per_step": total_ms / K, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": {"workload": CONFIG_TEXT[cfg_name], "config_id": cfg_name, "graph": synth.CONFIGS[cfg_name]["graph"],
                           "n_vertices": int(g["n_vertices"]), "n_arcs": int(len(g["src"])),
                           "objects": cfg["n_objects"], "updates_per_step": n_upd, "queries_per_step_per_gpu": Q,
                           "k": k, "cell_size": cs, "l2": "flushed between timed steps (256 MB write)",
                           "parallelism": (f"cell-ownership shards x{world} (one request/reply exchange per batch)"
                                           if shard else f"replicas x{world}, queries sharded")},
                "updates_per_s": updates_per_s, "per_kernel": per_kernel, "roofline": roofline,
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(st1["launches"]), "clocks": clk,
                "knn_rounds_per_step": (st1["knn_rounds"] - st0["knn_rounds"]) / K,
                "remote_requests_per_step_rank0": remote_requests / K if shard else None,
                "expand_work_per_query": {n: v / (Q * K) for n, v in dx.items()}, "delta": st1["delta"],
                "expand_promotions_per_step": (st1["expand_promotions"] - st0["expand_promotions"]) / K,
                "expand_retries_per_step": (st1["expand_retries"] - st0["expand_retries"]) / K}
        print(json.dumps(line), flush=True)
    grid.close()
    if world > 1:
        torch.distributed.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C1", choices=["C0", "C1", "C2", "C3"])
    ap.add_argument("--queries", type=int, default=0)
    ap.add_argument("--cell-size", type=int, default=0)
    ap.add_argument("--delta", type=int, default=0)
    ap.add_argument("--log-capacity", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=12)
    ap.add_argument("--ref-sample", type=int, default=400)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--parallel", default="shard", choices=["shard", "replicas"],
                    help="N>1 layout: cell-ownership shards (SURVEY 8(e)) or full replicas")
    args = ap.parse_args()
    assert args.warmup >= 3 or args.impl == "reference" or os.environ.get("BENCH_ALLOW_SHORT"), "W >= 3"
    if args.impl == "reference":
        run_reference(args, args.config)
    else:
        run_ours(args, args.config)


if __name__ == "__main__":
    main()
