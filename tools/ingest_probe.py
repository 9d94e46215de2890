"""Large-batch ingest timing (and an ncu target): C1 graph, |O| objects, batches of n updates
generated on the device.  Usage: python tools/ingest_probe.py [n_objects] [batch] [reps]"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icde_li0qhdy18_b200 as gg  # noqa: E402
import synth  # noqa: E402
from synth.device_walk import DeviceRandomWalk  # noqa: E402

n_obj = int(float(sys.argv[1])) if len(sys.argv) > 1 else 10_000
batch = int(float(sys.argv[2])) if len(sys.argv) > 2 else 10_000_000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
cfg = sys.argv[4] if len(sys.argv) > 4 else "C1"
g = synth.config_graph(cfg)
walk = DeviceRandomWalk(g, n_obj)
ticks = -(-batch // n_obj)
u = walk.ticks(ticks)[:batch].contiguous()
mode = int(os.environ.get("GG_INGEST_KERNELS", "0"))  # opts.ingest_kernels (3: three launches)
grid = gg.GGrid(g, 1024, max_objects=n_obj, profile=True, log_capacity=int(batch * (reps + 2) * 1.1),
                ingest_kernels=mode)
grid.ingest(u)
torch.cuda.synchronize()
grid.stats_reset()
for _ in range(reps):
    grid.ingest(u)
st = grid.stats()
km = st["kernel_ms"]
tot = sum(km[k] for k in ("ingest_classify", "ingest_alloc", "ingest_scatter"))
print(f"{cfg} mode={mode} |O|={n_obj} batch={batch}: classify {km['ingest_classify']/reps:.3f} alloc {km['ingest_alloc']/reps:.3f} "
      f"scatter {km['ingest_scatter']/reps:.3f} ms  -> {batch*reps/(tot/1e3)/1e9:.2f} G updates/s, "
      f"{48*batch*reps/(tot/1e3)/1e9:.0f} GB/s algorithmic")
