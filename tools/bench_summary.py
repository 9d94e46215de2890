"""One-line summary of a bench.py JSON line: python tools/bench_summary.py log [log...]"""
import json
import sys

for path in sys.argv[1:]:
    lines = [json.loads(x) for x in open(path) if x.startswith("{")]
    if not lines:
        print(path, "no JSON line")
        continue
    b = lines[-1]
    pk = {k: (round(v["ms_total"], 3), round(v["gbs"])) for k, v in b.get("per_kernel", {}).items()}
    w = {k: round(v, 1) for k, v in b.get("expand_work_per_query", {}).items()}
    print(f"{path}: value={b['value']:.4g} {b['unit']} ms/step={b['ms_per_step']:.3f} "
          f"e2e={b.get('e2e', {}).get('value', 0):.4g} kernels(ms,GB/s)={pk} work/q={w} "
          f"roof={b.get('roofline', {}).get('kernel')}:{b.get('roofline', {}).get('frac', 0):.3f} "
          f"rounds={b.get('knn_rounds_per_step')} clocks={b.get('clocks', {}).get('sm_mhz')}")
