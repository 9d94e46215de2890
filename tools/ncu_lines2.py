"""Per-CUDA-source-line warp-stall samples and instruction counts of one ncu report.

    python tools/ncu_lines2.py <report.ncu-rep> [top]
(ncu --page source --print-source cuda,sass: source lines with their SASS rows beneath.)"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname = "?"
agg = {}
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
    if r[0]:  # a source line row (aggregate of its SASS)
        try:
            smp = int(r[4] or 0)
            ins = int(r[7] or 0)
        except ValueError:
            continue
        agg[(fname, int(r[0]))] = (smp, ins, r[1][:100])
tot = sum(v[0] for v in agg.values()) or 1
print(f"total stall samples {tot}")
for (f, l), (s, i, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{100 * s / tot:5.1f}%  {f}:{l:<5d} inst {i:>11d}  {src}")
