"""Benchmark: kNN queries/s including the lazy flush at a fixed update rate (BASELINE.json).

One step = one pass of the whole hot path over one batch of synthetic input:
  ggrid_ingest(one tick of the random walk: every object reports once)   (Alg. 1: a0)
  ggrid_knn(Q queries, k)        (cell selection, lazy flush, expansion, candidate top-k,
                                  unresolved vertices, refinement: a1-a6 of SURVEY §8(a))
Default workload: BASELINE configs[3], the largest single-GPU config -- USA-shaped graph
(23,974,347 V / 58,333,344 arcs, Table II P@55786), 1M objects, 64 cached records per object
(64M records, >> L2) preloaded before the timed region, then per step 1M updates (f = 1 per
step, P@58136) and Q = 65,536 queries with k = 10.
value = queries answered / device time of the K steps (CUDA events on the library's stream,
max over ranks).  The line also carries:
  flush        a full flush of the 64M-record log (the flush kernel's HBM roofline, §8(d));
  roofline     the dominant kernel of the step (the expansion) against measured HBM, with its
               latency model and ncu limiters (it is latency/issue-bound);
  parity       the last timed step's answers vs the CPU oracle on sampled rows (bit-exact);
  cpu_baseline the oracle's early-exit mode on a bounded sample of the step's queries, and its
               serial latest-per-object pass as updates/s, with cores and CPU model;
  e2e          the same step through the public API from pinned host buffers (pipelined).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3|C0|C1|C2]
    python bench.py --impl reference ...    # the CPU oracle as the reference arm
Multi-GPU: --gpus N without a torchrun environment re-launches itself under torchrun with N
ranks.  Ranks own contiguous Z-order ranges of cells (cell-ownership sharding);
the global batch of Q queries is fixed and split across ranks (strong scaling); queries are
answered with one request/reply exchange that the library runs itself (ggrid.h "multi-GPU":
route, owner search, bounded requests, replies, merge, return -- kernels + NCCL send/recv).
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

CONFIG_TEXT = {  # BASELINE.json configs, verbatim
    "C0": "Fig.1-scale toy: ~1k-vertex synthetic grid road graph, 100 moving objects, 1k cached updates, k=3, 100 queries",
    "C1": "NY-shaped synthetic road graph (~264k vertices, ~734k edges), 10k objects, k=10, 1M cached updates",
    "C2": "FLA-shaped synthetic road graph (~1.07M vertices), 100k objects, k=10–50 sweep",
    "C3": "USA-shaped synthetic road graph (~24M vertices, ~58M edges), 1M objects, k=10, batched queries on 1/2/4/8 GPUs",
}
METRIC = "kNN queries/sec incl. lazy flush at fixed update rate; updates/sec; HBM GB/s"
SEEDS = {"graph": synth.SEED_GRAPH, "objects": synth.SEED_OBJECTS, "updates": synth.SEED_UPDATES,
         "queries": synth.SEED_QUERIES}

# Algorithmic bytes per unit (restated in DESIGN.md §4)
INGEST_BYTES_PER_UPDATE = 48          # 16 record + 4 arc->cell + 8 RED.MAX + 20 SoA write
FLUSH_BYTES_PER_RECORD = 12           # obj + key (the ot_key match is an L1-resident gather)
FLUSH_BYTES_PER_WINNER = 12 + 24 + 8 + 12  # payload read + compacted write + v_obj set + (next flush) clear
# query (§8(d) "Query, per query"): ball vertices x (4 rowptr + 4 D) + ball arcs x 8 (col + w)
# + objects read x 12 + 8k output; the kernel counts the vertices, arcs and objects it touches
EXPAND_BYTES_PER_VERTEX = 8
EXPAND_BYTES_PER_ARC = 8
EXPAND_BYTES_PER_OBJECT = 12
# latency model of the expansion: per delta-stepping round, three dependent
# global-memory trips (frontier vertex's inline arcs / cell state -> its object records ->
# their ot_key validity) at the L2 hit latency, plus the round's two CTA barriers and shared-
# memory table work; a query is one chain of rounds; resident queries run concurrently
L2_HIT_CYCLES = 250            # B300_MICROARCH.md "L2 hit latency" 234 near-die / 262 far-die
ROUND_TRIPS = 3
ROUND_ONCHIP_CYCLES = 300      # 2 barriers + partition + LDS/ATOMS chain per round (estimate)

# opts.profile masks (include/ggrid.h): bit 0 = every launch kind, bit k+1 = kind k.  A timed
# launch costs a few us of device idle time, so the timed steps time only the dominant kernel
# (the expansion, GGRID_K_EXPAND = 5 / GGRID_K_EXPAND_BIG = 6); the per-kernel split comes from
# extra, untimed breakdown steps with every launch timed.
PROFILE_ALL = 1
PROFILE_EXPAND = (2 << 5) | (2 << 6)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)", float(d.get("sm_max_mhz", 1965.0))
    return 7672.0, "fallback (B200_PROFILING.md)", 1965.0


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor() or "unknown"


def workload(cfg: str, queries: int | None):
    c = dict(synth.CONFIGS[cfg])
    c.update(synth.BENCH_STEPS[cfg])
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
        self.mark_rows = 0
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(gpu), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "20"],
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
        timed = rows[self.mark_rows:]
        if timed:
            rows = timed
        else:  # a timed region shorter than the 20 ms sampling interval: the warm-up's last samples
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


# -------------------------------------------------------------------------- oracle timing
def oracle_query_rate(g, ids, e, d, queries, k, n_small, n_large, threads=0):
    """Early-exit oracle (the §8(d) timing mode) queries/s on the host cores, as it stands.
    Each oracle call rebuilds its CSR and object index, so two calls on nested samples are
    timed and the rate is their marginal one: (n_large - n_small) / (t_large - t_small).
    Returns (rate, answers of the first n_small queries, detail dict)."""
    import oracle

    cores = threads if threads > 0 else oracle.hardware_threads()
    t0 = time.perf_counter()
    so, sd = oracle.knn(g, ids, e, d, queries[:n_small], k, mode=oracle.EARLY, threads=cores)
    t_small = time.perf_counter() - t0
    t0 = time.perf_counter()
    oracle.knn(g, ids, e, d, queries[:n_large], k, mode=oracle.EARLY, threads=cores)
    t_large = time.perf_counter() - t0
    rate = (n_large - n_small) / max(1e-9, t_large - t_small)
    return rate, (so, sd), {"cores": cores, "t_small_s": t_small, "t_large_s": t_large,
                            "n_small": n_small, "n_large": n_large}


def oracle_update_rate(upd, n_obj, seen_before):
    """The oracle's serial latest-per-object pass (§8(c) step 1) on one step's updates."""
    import oracle

    snap = oracle.Snapshot(n_obj)
    snap.n_seen = seen_before
    t0 = time.perf_counter()
    snap.apply(upd)
    return len(upd) / max(1e-9, time.perf_counter() - t0)


# -------------------------------------------------------------------------- reference arm
def run_reference(args, cfg_name):
    """The CPU oracle as the reference arm: each step is a bounded sample of the workload --
    the serial snapshot pass over the step's updates and the early-exit oracle on
    args.ref_sample of the step's queries (graph CSR build included, as the oracle stands)."""
    world, rank, _ = dist_setup()
    if world > 1 and rank != 0:
        return
    import oracle

    cfg = workload(cfg_name, args.queries)
    g = synth.config_graph(cfg_name)
    walk = synth.RandomWalk(g, cfg["n_objects"])
    snap = oracle.Snapshot(cfg["n_objects"])
    snap.apply(walk.ticks(cfg["preload_ticks"]))  # the cached log (untimed, like our preload)
    cores = oracle.hardware_threads()
    S = min(args.ref_sample, cfg["n_queries"])
    times = []
    for s in range(args.warmup + args.steps):
        upd = walk.ticks(cfg["step_ticks"])
        q = synth.queries(g, cfg["n_queries"], seed=synth.SEED_QUERIES + s)[:S]
        t0 = time.perf_counter()
        snap.apply(upd)
        ids, e, d = snap.objects()
        oracle.knn(g, ids, e, d, q, cfg["k"], mode=oracle.EARLY, threads=cores)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            times.append(dt)
    value = S * len(times) / sum(times)
    sample = (f"per step: the serial latest-per-object pass over the step's {len(upd)} updates + the "
              f"early-exit oracle (its CSR build included) on {S} of the step's {cfg['n_queries']} queries")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic", "seeds": SEEDS,
            "config": {"workload": CONFIG_TEXT[cfg_name], "config_id": cfg_name,
                       "queries_per_step": S, "updates_per_step": len(upd), "k": cfg["k"]},
            "cpu_baseline": {"value": value, "unit": "queries/s", "cores": cores, "cpu": cpu_model(),
                             "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def run_ours(args, cfg_name):
    import torch

    import paper_conf_icde_li0qhdy18_b200 as gg
    from paper_conf_icde_li0qhdy18_b200 import dist as gdist

    world, rank, local = dist_setup()
    backend = os.environ.get("BENCH_DIST_BACKEND", "nccl")
    if world > 1:
        import torch.distributed as dist

        # one process per GPU over NCCL; BENCH_DIST_BACKEND=gloo lets the harness be exercised
        # with several ranks sharing one GPU (a test mode, not a measurement)
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
    Q, k, n_obj = cfg["n_queries"], cfg["k"], cfg["n_objects"]
    cell_size = args.cell_size or cfg["cell_size"]
    lo, hi = gdist.shard_range(Q, rank, world)  # this rank's share of the global batch
    Qr = hi - lo
    shard = world > 1 and args.parallel == "shard"
    t_setup = time.perf_counter()
    g = synth.config_graph(cfg_name)
    walk = synth.RandomWalk(g, n_obj)
    n_step_upd = n_obj * cfg["step_ticks"]
    preload = walk.ticks(cfg["preload_ticks"]) if cfg["preload_ticks"] else np.empty((0, 4), np.uint32)
    # the record arena: superseded extents are reclaimed by a garbage collection when it fills;
    # 2^29 records (12.9 GB of 180) keep the setup's three re-ingested 64M-record flushes and
    # ~160 steps after them (2M records per C3 step) collection-free (amortised, reported)
    log_cap = args.log_capacity or max(1 << 29, int(1.25 * (len(preload) + 8 * n_step_upd)) + (1 << 20))
    hist = [preload]  # every update the index has seen, in arrival order (for the parity check)

    n_break = max(3, min(args.steps, 10))  # breakdown steps (every launch timed), after the timed ones
    n_steps_total = args.warmup + args.steps + n_break
    step_u, step_q = [], []
    for s in range(n_steps_total):
        u = walk.ticks(cfg["step_ticks"])
        step_u.append(u)
        step_q.append(synth.queries(g, Q, seed=synth.SEED_QUERIES + s)[lo:hi])
    t_gen = time.perf_counter() - t_setup

    # cell-ownership sharding: this rank's handle is shard `rank` of `world` and
    # the library runs the query exchange itself (ggrid.h "multi-GPU"): over NCCL between GPUs,
    # over a gloo all-to-all callback in the one-GPU harness mode (BENCH_DIST_BACKEND=gloo)
    shard_opts = {}
    if shard:
        if backend == "nccl":
            uid = [gg.ggrid_nccl_unique_id() if rank == 0 else None]
            torch.distributed.broadcast_object_list(uid, src=0)
            shard_opts = dict(n_ranks=world, rank=rank, nccl_id=uid[0])
        else:
            shard_opts = dict(n_ranks=world, rank=rank, exchange=gg.alltoall_callback())
    stream = torch.cuda.Stream()
    t0 = time.perf_counter()
    grid = gg.GGrid(g, cell_size, max_objects=n_obj, profile=PROFILE_ALL, log_capacity=log_cap,
                    delta=args.delta, stream=stream.cuda_stream, async_ingest=True, **shard_opts)
    t_build = time.perf_counter() - t0
    out_o = torch.empty((Qr, k), dtype=torch.int32, device="cuda")
    out_d = torch.empty((Qr, k), dtype=torch.int32, device="cuda")
    # > 126 MB L2
    l2 = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    peak, peak_src, sm_mhz_max = load_peaks()

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()

    # ---- preload (untimed) + the flush sub-record: full flushes of the cached log ----------
    flush_rec = None
    if len(preload):
        dpre = torch.from_numpy(preload.view(np.int32)).to("cuda")
        rounds = []
        n_rounds = 3
        for r in range(n_rounds):
            grid.stats_reset()
            s0 = grid.stats()
            grid.ingest(dpre)  # the same records again in later rounds: newer arrivals, same locations
            grid.sync()
            s1 = grid.stats()
            ing_ms = sum(s1["kernel_ms"][x] for x in ("ingest_classify", "ingest_alloc", "ingest_scatter"))
            with torch.cuda.stream(stream):
                l2.zero_()
            grid.stats_reset()
            s1 = grid.stats()
            grid.flush_all()
            s2 = grid.stats()
            rec = s2["records_flushed"] - s1["records_flushed"]
            win = s2["objects_written"] - s1["objects_written"]
            fms = s2["kernel_ms"]["flush"]
            alg = rec * FLUSH_BYTES_PER_RECORD + win * FLUSH_BYTES_PER_WINNER
            rounds.append(dict(flush_ms=fms, records=rec, winners=win, cells=s2["cells_flushed"] - s1["cells_flushed"],
                               alg_bytes=alg, gbs=alg / (fms / 1e3) / 1e9, ingest_ms=ing_ms,
                               ingest_updates_per_s=len(preload) / (ing_ms / 1e3)))
        hist += [preload] * (n_rounds - 1)  # (re-ingested: later arrivals of the same records)
        med = sorted(rounds, key=lambda x: x["flush_ms"])[len(rounds) // 2]
        flush_rec = {"records": med["records"], "winners": med["winners"], "cells": med["cells"],
                     "ms": med["flush_ms"], "alg_bytes": med["alg_bytes"], "achieved_gbs": med["gbs"],
                     "peak_gbs": peak, "frac": med["gbs"] / peak, "spec_gbs": 8000.0,
                     "frac_of_spec": med["gbs"] / 8000.0, "bound": "hbm",
                     "bytes_model": "12 B per cached record (obj + key) + 56 B per surviving object",
                     "timing": f"CUDA events around each flush launch, median of {n_rounds} full flushes "
                               "(each after re-ingesting the whole log; L2 flushed before each)",
                     "bulk_ingest_updates_per_s": sorted(x["ingest_updates_per_s"] for x in rounds)[len(rounds) // 2],
                     "bulk_ingest_batch": len(preload)}
        del dpre
    grid.set_profile(PROFILE_EXPAND)

    # ---- device-resident timed region -------------------------------------------------------
    times = []
    st0 = st1 = sb0 = None
    clk = None
    last_out = None
    for s in range(n_steps_total):
        u = step_u[s]
        if rank == 0:  # the update stream arrives at rank 0 and is fanned out over NCCL
            du = torch.from_numpy(u.view(np.int32)).to("cuda")
        else:
            du = torch.empty((len(u), 4), dtype=torch.int32, device="cuda")
        dq = torch.from_numpy(step_q[s].view(np.int32)).to("cuda")
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
                gdist.broadcast_updates(du, src=0)
            grid.ingest(du)
            grid.knn(dq, k, out_o, out_d)  # (sharded: collective over the ranks, inside the library)
            e1.record(stream)
        e1.synchronize()
        hist.append(u)
        if args.warmup <= s < args.warmup + args.steps:
            times.append(e0.elapsed_time(e1))
        if s == args.warmup + args.steps - 1:  # the last timed step's answers, for the parity check
            last_out = (out_o.cpu().numpy().view(np.uint32).copy(), out_d.cpu().numpy().view(np.uint32).copy(),
                        len(hist))
    barrier()
    grid.sync()
    sb1 = grid.stats()
    total_ms = gdist.max_over_ranks(sum(times), device="cuda")
    req_all = 0.0
    if shard:  # bounded requests sent over the timed steps, summed over the ranks
        t_req = torch.tensor([float(st1["remote_requests"] - st0["remote_requests"])], dtype=torch.float64, device="cuda")
        torch.distributed.all_reduce(t_req)
        req_all = float(t_req.item())
    K = args.steps
    value = Q * K / (total_ms / 1e3)  # the global batch Q per step, all ranks (max-over-ranks time)

    # ---- per-kernel split and the dominant kernel's roofline -----------------------------------
    def kernels(a, b, nsteps):
        kms, kl = b["kernel_ms"], b["kernel_launches"]
        rec = b["records_flushed"] - a["records_flushed"]
        win = b["objects_written"] - a["objects_written"]
        dx = {n: b["expand_" + n] - a["expand_" + n] for n in ("iterations", "vertices", "arcs", "harvested", "objects")}
        nq = Qr * nsteps
        expand_bytes = (dx["vertices"] * EXPAND_BYTES_PER_VERTEX + dx["arcs"] * EXPAND_BYTES_PER_ARC
                        + dx["objects"] * EXPAND_BYTES_PER_OBJECT + nq * 8 * k)
        kern = {
            "ingest": (kms["ingest_classify"] + kms["ingest_alloc"] + kms["ingest_scatter"],
                       n_step_upd * nsteps * INGEST_BYTES_PER_UPDATE,
                       kl["ingest_classify"] + kl["ingest_alloc"] + kl["ingest_scatter"]),
            "flush": (kms["flush"], rec * FLUSH_BYTES_PER_RECORD + win * FLUSH_BYTES_PER_WINNER, kl["flush"]),
            # (level-0 launches: the chained level above runs beside them, inside their event pair)
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
                "traffic": traffic, "kernel": dom, "peak_source": peak_src,
                "launch_ms": dms / max(1, dl), "launches": dl,
                "timed_in": "timed steps" if dom == "expand" else "breakdown steps",
                "bytes_model": "SURVEY 8(d) per query: expanded vertices x 8 + relaxed arcs x 8 + objects read x 12 + 8k"}
    if dom == "expand":
        nq = Qr * K
        rounds_q = dx["iterations"] / max(1, nq)
        # the C3 starting level: the one-warp kernel with its narrow table, 8 CTAs x 4 queries per
        # SM (shared memory and 64 registers), less the few CTAs reserved for the chained level
        sms = torch.cuda.get_device_properties(dev).multi_processor_count
        resident = int(os.environ.get("BENCH_EXPAND_RESIDENT", str(sms * 32)))
        cyc = rounds_q * (ROUND_TRIPS * L2_HIT_CYCLES + ROUND_ONCHIP_CYCLES)
        t_model_ms = nq / resident * cyc / (sm_mhz_max * 1e3)
        roofline["latency_model"] = {
            "rounds_per_query": rounds_q, "dependent_l2_trips_per_round": ROUND_TRIPS,
            "l2_hit_cycles": L2_HIT_CYCLES, "onchip_cycles_per_round": ROUND_ONCHIP_CYCLES,
            "resident_queries": resident, "model_ms": t_model_ms, "measured_ms": dms,
            "frac": t_model_ms / dms if dms > 0 else None}
    lp = os.path.join(ROOT, "profiles", f"limiters_{cfg_name}.json")
    if os.path.exists(lp):  # what bounds the kernel when it is not HBM (ncu, the last profiling pass)
        lim = json.load(open(lp)).get(dom)
        roofline["ncu_limiters"] = lim
        if lim and lim.get("warp_instructions") and dom == "expand":
            # issue roofline: the capture's warp instructions per query, issued at one per
            # scheduler per cycle (148 SMs x 4 schedulers at the max clock), for this run's queries
            inst_q = lim["warp_instructions"] / max(1, cfg["n_queries"] // world)
            t_issue_ms = inst_q * Qr * K / (148 * 4 * sm_mhz_max * 1e6) * 1e3
            roofline["issue_model"] = {"warp_instructions_per_query": inst_q, "schedulers": 148 * 4,
                                       "clock_mhz": sm_mhz_max, "model_ms": t_issue_ms, "measured_ms": dms,
                                       "frac": t_issue_ms / dms if dms > 0 else None,
                                       "source": "ncu smsp__inst_executed.sum of one launch (profiles/limiters_C3.json)"}
    updates_per_s = n_step_upd * K / (ingest_ms / 1e3) if ingest_ms > 0 else None

    # ---- parity of the last timed step (rank 0's share) against the oracle -------------------
    parity = None
    cpu = None
    if rank == 0 and not args.no_parity:
        import oracle

        go, gd, n_hist = last_out
        snap = oracle.Snapshot(n_obj)
        for u in hist[:n_hist]:
            snap.apply(u)
        ids, e_, d_ = snap.objects()
        qs = step_q[args.warmup + args.steps - 1]
        S = min(args.parity_rows, Qr)
        sel = np.linspace(0, Qr - 1, S).astype(np.int64)
        rng = np.random.default_rng(7)
        sel = np.unique(np.concatenate([sel, rng.choice(Qr, size=min(S, Qr), replace=False)]))[:max(S, 1)]
        t0 = time.perf_counter()
        ro, rd = oracle.knn(g, ids, e_, d_, qs[sel], k, mode=oracle.EARLY)
        t_early = time.perf_counter() - t0
        ok_rows = (go[sel] == ro).all(1) & (gd[sel] == rd).all(1)
        nf = min(args.parity_full, len(sel))
        t0 = time.perf_counter()
        fo, fd = oracle.knn(g, ids, e_, d_, qs[sel[:nf]], k, mode=oracle.FULL)
        t_full = time.perf_counter() - t0
        ok_full = (go[sel[:nf]] == fo).all(1) & (gd[sel[:nf]] == fd).all(1)
        parity = {"rows": int(len(sel)), "rows_exact": int(ok_rows.sum()), "exact": bool(ok_rows.all() and ok_full.all()),
                  "oracle_mode": "early-exit (exact, cross-checked against full on the first rows)",
                  "full_dijkstra_rows": int(nf), "full_dijkstra_exact": int(ok_full.sum()),
                  "step": args.warmup + args.steps - 1, "rank": rank, "seconds": t_early + t_full,
                  "bar": "bit-exact object ids and distances, ties by id"}
        # ---- CPU oracle beside it (rank 0, N = 1 only): a bounded sample of the step -------------
        if world == 1 and not args.no_cpu_baseline:
            n_small = min(args.cpu_small, Qr)
            n_large = min(args.cpu_sample, Qr)
            qrate, _, det = oracle_query_rate(g, ids, e_, d_, qs, k, n_small, n_large)
            urate = oracle_update_rate(step_u[-1], n_obj, 0)
            cpu = {"value": qrate, "unit": "queries/s", "cores": det["cores"], "cpu": cpu_model(), "kind": "oracle",
                   "sample": (f"early-exit oracle (threads = cores, one query per task) on the first {n_large} and "
                              f"{n_small} queries of the last timed step's batch, after its snapshot; rate = "
                              f"({n_large}-{n_small}) / ({det['t_large_s']:.2f}s - {det['t_small_s']:.2f}s) (the "
                              f"difference cancels each call's CSR build)"),
                   "updates_per_s": urate,
                   "updates_sample": f"serial latest-per-object pass over one step's {len(step_u[-1])} updates"}

    # ---- e2e through the public API with pinned host buffers -------------------------------
    # Pipelined (ggrid_ingest_stage / ggrid_query_stage, then ggrid_ingest_commit /
    # ggrid_knn_commit, P@45017-45625): the next step's update and query batches are copied from
    # pinned host memory while this step's queries run.  The timed region holds every step's H2D
    # copies, the ingest, the queries and the D2H of the answers.  A fresh index without
    # profile-mode events (an event queued behind a staged copy costs ~50 us), preloaded and
    # flushed like the first (untimed).
    grid.close()
    if shard and backend == "nccl":  # a fresh communicator for the fresh index
        uid = [gg.ggrid_nccl_unique_id() if rank == 0 else None]
        torch.distributed.broadcast_object_list(uid, src=0)
        shard_opts["nccl_id"] = uid[0]
    grid = gg.GGrid(g, cell_size, max_objects=n_obj, log_capacity=log_cap, delta=args.delta, async_ingest=True,
                    **shard_opts)
    if len(preload):
        grid.ingest(torch.from_numpy(preload.view(np.int32)).to("cuda"))
        grid.flush_all()
    h_o = torch.empty((Qr, k), dtype=torch.int32).pin_memory()
    h_d = torch.empty((Qr, k), dtype=torch.int32).pin_memory()

    def e2e_stage(hu, hq):
        if shard:  # (the staged calls are single-shard; a sharded rank ingests directly)
            grid.ingest(hu)
            return
        grid.ingest_stage(hu)
        grid.query_stage(hq)  # copied behind the update batch on the library's copy stream

    def e2e_knn(hq):
        if not shard:
            grid.knn_commit(k, h_o, h_d)  # the staged queries; answers written to pinned memory in place
            return
        grid.knn(hq, k, h_o, h_d)  # (collective; the library copies the pinned batch in and out)

    n_e2e = max(1, args.e2e_steps)
    w_e2e = 3
    hus, hqs = [], []
    for s in range(w_e2e + n_e2e):
        u = step_u[s % len(step_u)]
        hus.append(torch.from_numpy(u.view(np.int32)).pin_memory())
        hqs.append(torch.from_numpy(step_q[s % len(step_q)].view(np.int32)).pin_memory())
    # one untimed DMA from every pinned input buffer (a producer reuses a fixed set of pinned
    # buffers; the first DMA from a freshly pinned allocation is measurably slower)
    scratch_u = torch.empty_like(hus[0], device="cuda")
    scratch_q = torch.empty_like(hqs[0], device="cuda")
    for hu, hq in zip(hus, hqs):
        scratch_u.copy_(hu)
        scratch_q.copy_(hq)
    torch.cuda.synchronize()
    del scratch_u, scratch_q
    def e2e_commit():
        if not shard:
            grid.ingest_commit()

    for s in range(w_e2e):  # warm-up steps
        e2e_stage(hus[s], hqs[s])
        e2e_commit()
        e2e_knn(hqs[s])
    hus, hqs = [None] + hus[w_e2e:], [None] + hqs[w_e2e:]
    barrier()
    t0 = time.perf_counter()
    e2e_stage(hus[1], hqs[1])
    for s in range(1, n_e2e + 1):
        e2e_commit()
        if s + 1 <= n_e2e:
            e2e_stage(hus[s + 1], hqs[s + 1])  # overlaps the queries below
        e2e_knn(hqs[s])
    grid.sync()  # (the last step's answers were read back inside knn already)
    e2e_total = gdist.max_over_ranks(time.perf_counter() - t0, device="cuda")
    e2e = {"value": Q * n_e2e / e2e_total, "unit": "queries/s",
           "h2d_bytes_per_step": n_step_upd * 16 + Qr * 8, "d2h_bytes_per_step": Qr * k * 8,
           "steps": n_e2e, "timing": "wall clock of the pipelined loop (stage/commit), max over ranks"}
    st_e = grid.stats()
    grid.close()

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": world, "steps": K,
                "warmup": args.warmup, "ms_per_step": total_ms / K, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u32",
                "data": "synthetic", "seeds": SEEDS,
                "config": {"workload": CONFIG_TEXT[cfg_name], "config_id": cfg_name,
                           "graph": synth.CONFIGS[cfg_name]["graph"],
                           "n_vertices": int(g["n_vertices"]), "n_arcs": int(len(g["src"])),
                           "objects": n_obj, "cached_records_preloaded": int(len(preload)),
                           "updates_per_step": n_step_upd, "queries_per_step": Q, "queries_per_step_rank0": Qr,
                           "k": k, "cell_size": int(st1["cell_size"]), "n_cells": int(st1["n_cells"]),
                           "l2": "flushed between timed steps (256 MB write); C3's log (1.5 GB) >> L2",
                           "parallelism": (f"cell-ownership shards x{world}, fixed global batch (one request/reply "
                                           "exchange per batch)" if shard else
                                           (f"replicas x{world}, global batch split" if world > 1 else "single GPU"))},
                "updates_per_s": updates_per_s, "flush": flush_rec, "per_kernel": per_kernel, "roofline": roofline,
                "parity": parity, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(st1["launches"]),
                "clocks": clk,
                "knn_rounds_per_step": (st1["knn_rounds"] - st0["knn_rounds"]) / K,
                "exchange": ({"kind": "nccl" if backend == "nccl" else "gloo all-to-all callback (harness mode)",
                              "requests_per_step_all_ranks": req_all / K} if shard else None),
                "expand_work_per_query": {n: v / (Qr * K) for n, v in dx.items()}, "delta": st1["delta"],
                "expand_promotions_per_step": (st1["expand_promotions"] - st0["expand_promotions"]) / K,
                "expand_retries_per_step": (st1["expand_retries"] - st0["expand_retries"]) / K,
                "gc_runs": int(sb1["gc_runs"]), "e2e_gc_runs": int(st_e["gc_runs"]),
                "setup_s": {"inputs": t_gen, "build": t_build}}
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def self_launch(args):
    """--gpus N outside torchrun: re-run this script under torchrun with N ranks (one per GPU).
    NCCL's communicator-init log lines are switched on so the ranks can be counted."""
    import socket

    with socket.socket() as s_:
        s_.bind(("127.0.0.1", 0))
        port = s_.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C3", choices=["C0", "C1", "C2", "C3"])
    ap.add_argument("--queries", type=int, default=0)
    ap.add_argument("--cell-size", type=int, default=0)
    ap.add_argument("--delta", type=int, default=0)
    ap.add_argument("--log-capacity", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=12)
    ap.add_argument("--ref-sample", type=int, default=1024, help="reference arm: queries per step")
    ap.add_argument("--cpu-sample", type=int, default=2048, help="cpu_baseline: larger early-exit sample")
    ap.add_argument("--cpu-small", type=int, default=256, help="cpu_baseline: smaller early-exit sample")
    ap.add_argument("--parity-rows", type=int, default=256)
    ap.add_argument("--parity-full", type=int, default=4)
    ap.add_argument("--no-parity", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--parallel", default="shard", choices=["shard", "replicas"],
                    help="N>1 layout: cell-ownership shards (SURVEY 8(e)) or full replicas")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        sys.exit(self_launch(args))
    assert args.warmup >= 3 or args.impl == "reference" or os.environ.get("BENCH_ALLOW_SHORT"), "W >= 3"
    if args.impl == "reference":
        run_reference(args, args.config)
    else:
        run_ours(args, args.config)


if __name__ == "__main__":
    main()
