"""Summarise an ncu 'cuda,sass' source page: samples and executed instructions per CUDA line.
usage: ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > s.csv; python tools/ncu_lines.py s.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
fname = ""
agg = []
hdr = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or r[0] in ("Function Name",):
        continue
    if r[2] != "-":  # sass row
        continue
    try:
        s = int(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
        ie = int(r[hdr.index("Instructions Executed")] or 0)
    except (ValueError, IndexError):
        continue
    agg.append((s, ie, fname, r[0], r[1].strip()[:100]))
ts = sum(a[0] for a in agg) or 1
ti = sum(a[1] for a in agg) or 1
print(f"total samples {ts}  warp-instructions {ti}")
for a in sorted(agg, reverse=True)[:top]:
    print(f"{a[0]:7d} {100 * a[0] / ts:5.1f}%  inst {100 * a[1] / ti:5.1f}%  {a[2]}:{a[3]:5s} {a[4]}")
