"""Summarise a profiling pass (tools/profile_round.sh) into profiles/<tag>_*.

    python tools/summarize_profiles.py r01

Writes profiles/<tag>_summary.md (per-kernel ncu metrics, stall reasons, launch-list shares),
profiles/<tag>_launches_C1.csv (the launch list), profiles/<tag>_<kernel>_raw.csv (ncu raw page
of each full capture) and profiles/traffic_<cfg>.json (DRAM bytes per launch of each kernel,
read by bench.py for the roofline `traffic` field).
"""
import collections
import csv
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
src = os.path.join(ROOT, "gpurun_out", f"prof_{tag}")
dst = os.path.join(ROOT, "profiles")
os.makedirs(dst, exist_ok=True)

WANT = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit rate"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active % (achieved occupancy)"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__occupancy_limit_registers", "CTA limit (registers)"),
    ("launch__occupancy_limit_shared_mem", "CTA limit (smem)"),
]


def raw_rows(path):
    rows = list(csv.reader(open(path)))
    hdr, units = rows[0], rows[1]
    return [(hdr, units, r) for r in rows[2:]]


lines = [f"# Profiling summary — round tag `{tag}`", "",
         "Source: `tools/profile_c3.sh` (earlier rounds: `tools/profile_round.sh`) under gpurun on one B200 (ncu 2025, `--clock-control none`).",
         "Raw pages: `profiles/%s_<capture>_raw.csv`; launch list: `profiles/%s_launches_C1.csv`." % (tag, tag), ""]
traffic = {}
issue = {}
caps = sorted(f[:-len("_raw.csv")] for f in os.listdir(src) if f.endswith("_raw.csv"))
for cap in caps:
    p = os.path.join(src, f"{cap}_raw.csv")
    shutil.copy(p, os.path.join(dst, f"{tag}_{cap}_raw.csv"))
    for hdr, units, r in raw_rows(p):
        name = r[hdr.index("Kernel Name")].split("(")[0]
        lines.append(f"## `{name}` ({cap})")
        lines.append("")
        lines.append("| metric | value |")
        lines.append("|---|---|")
        for key, label in WANT:
            if key in hdr:
                i = hdr.index(key)
                lines.append(f"| {label} (`{key}`) | {r[i]} {units[i]} |")
        stalls = []
        for i, k in enumerate(hdr):
            if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("_not_issued"):
                try:
                    stalls.append((float(r[i].replace(",", "")), k.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        tot = sum(v for v, _ in stalls) or 1.0
        top = ", ".join(f"{n} {100 * v / tot:.0f}%" for v, n in sorted(stalls, reverse=True)[:6])
        lines.append(f"| warp stall samples (top) | {top} |")
        lines.append("")
        rd = float(r[hdr.index("dram__bytes_read.sum")].replace(",", ""))
        wr = float(r[hdr.index("dram__bytes_write.sum")].replace(",", ""))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rd *= scale.get(units[hdr.index("dram__bytes_read.sum")], 1)
        wr *= scale.get(units[hdr.index("dram__bytes_write.sum")], 1)
        kind, cfg = cap.rsplit("_", 1)
        kind = {"ingestscatter": "ingest_bulk_scatter", "ingestclassify": "ingest_bulk_classify",
                "stepscatter": "ingest_step_scatter", "stepingest": "ingest_step",
                "stepflush": "flush_step"}.get(kind, kind)
        traffic.setdefault(cfg, collections.defaultdict(float))[kind] += rd + wr
        if "smsp__issue_active.avg.pct_of_peak_sustained_active" in hdr:  # (non-HBM limiters)
            issue.setdefault(cfg, {})[kind] = {
                "issue_slots_busy_pct": float(r[hdr.index("smsp__issue_active.avg.pct_of_peak_sustained_active")]),
                "warp_instructions": float(r[hdr.index("smsp__inst_executed.sum")].replace(",", "")),
                "duration_ns": float(r[hdr.index("gpu__time_duration.sum")].replace(",", "")) * (
                    1e3 if units[hdr.index("gpu__time_duration.sum")] == "us" else
                    1e6 if units[hdr.index("gpu__time_duration.sum")] == "ms" else 1.0),
                "dram_throughput_pct": float(r[hdr.index("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed")]),
                "top_stalls": top, "capture": f"profiles/{tag}_summary.md"}

for ll in [os.path.join(src, f) for f in sorted(os.listdir(src)) if f.startswith("launches_") and f.endswith(".csv")]:
    lcfg = os.path.basename(ll)[len("launches_"):-4]
    shutil.copy(ll, os.path.join(dst, f"{tag}_launches_{lcfg}.csv"))
    rows = list(csv.reader(open(ll)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    agg = collections.defaultdict(list)
    for r in rows[hi + 1:]:
        agg[r[h.index("Kernel Name")].split("(")[0]].append(float(r[h.index("Metric Value")].replace(",", "")))
    tot = sum(sum(v) for k, v in agg.items() if "gg::" in k)
    lines += [f"## Launch list, bench ({lcfg}), cold-cache serialised (`gpu__time_duration.sum`)", "",
              "| kernel | launches | mean µs | share of library time |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
        share = f"{100 * sum(v) / tot:.1f}%" if "gg::" in k else "(torch L2 flush, untimed)"
        lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {share} |")
    lines.append("")
    # the bench steps alone (from the first step ingest on; the setup's bulk ingests and full
    # flushes excluded): the share each kernel takes of a step, to compare with the bench's
    # CUDA-event split
    names = [r[h.index("Kernel Name")].split("(")[0] for r in rows[hi + 1:]]
    vals = [float(r[h.index("Metric Value")].replace(",", "")) for r in rows[hi + 1:]]
    first = next((i for i, n in enumerate(names) if "k_ingest_direct" in n or "k_ingest_fused" in n), None)
    if first is not None:  # (up to the e2e section's fresh index: its bulk preload ingest)
        end = next((i for i in range(first, len(names))
                    if "k_ingest_classify" in names[i] or "k_bulk_keys" in names[i]), len(names))
        st = collections.defaultdict(list)
        for n, v in zip(names[first:end], vals[first:end]):
            if "gg::" in n:
                st[n].append(v)
        tot = sum(sum(v) for v in st.values())
        lines += [f"## Launch list, bench steps only ({lcfg}): share of the step", "",
                  "| kernel | launches | mean µs | share of the step's library time |", "|---|---|---|---|"]
        for k, v in sorted(st.items(), key=lambda x: -sum(x[1])):
            lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {100 * sum(v) / tot:.1f}% |")
        lines.append("")

open(os.path.join(dst, f"{tag}_summary.md"), "w").write("\n".join(lines) + "\n")
for cfg, d in traffic.items():
    # per launch: expand (the starting level), ingest (one fused launch per step), flush (C3)
    json.dump({k: v for k, v in d.items()}, open(os.path.join(dst, f"traffic_{cfg}.json"), "w"), indent=1)
for cfg, d in issue.items():
    json.dump(d, open(os.path.join(dst, f"limiters_{cfg}.json"), "w"), indent=1)
print("\n".join(lines))
