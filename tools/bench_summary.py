"""One-line summary of a bench.py JSON line: python tools/bench_summary.py log [log...]"""
import json
import sys

for path in sys.argv[1:]:
    lines = [json.loads(x) for x in open(path) if x.startswith("{")]
    if not lines:
        print(path, "no JSON line")
        continue
    b = lines[-1]
    pk = {k: (round(v.get("ms_per_step", v.get("ms_total", 0)), 4), round(v["gbs"]))
          for k, v in b.get("per_kernel", {}).items() if isinstance(v, dict)}
    w = {k: round(v, 1) for k, v in b.get("expand_work_per_query", {}).items()}
    print(f"{path}: value={b['value']:.4g} {b['unit']} ms/step={b['ms_per_step']:.3f} "
          f"e2e={b.get('e2e', {}).get('value', 0):.4g} kernels(ms,GB/s)={pk} work/q={w} "
          f"roof={b.get('roofline', {}).get('kernel')}:{b.get('roofline', {}).get('frac', 0):.3f} "
          f"launch_ms={b.get('roofline', {}).get('launch_ms', 0):.4f} "
          f"L0={b['per_kernel']['expand'].get('level0_ms_per_step', 0):.4f} Lhi={b['per_kernel']['expand'].get('higher_levels_ms_per_step', 0):.4f} "
          f"parity={(b.get('parity') or {}).get('rows_exact')}/{(b.get('parity') or {}).get('rows')} "
          f"rounds={b.get('knn_rounds_per_step')} promo={b.get('expand_promotions_per_step')} retry={b.get('expand_retries_per_step')} clocks={b.get('clocks', {}).get('sm_mhz')}")
