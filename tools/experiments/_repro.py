import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_icde_li0qhdy18_b200 as gg, synth
g = synth.table_ii_graph("NY", scale=0.2)
upd = synth.RandomWalk(g, 20_000, inject=True).ticks(30)
for mode in (0, 3):
  for it in range(3):
    grid = gg.GGrid(g, 256, max_objects=20_000, ingest_kernels=mode)
    grid.ingest(upd)
    q = synth.queries(g, 400)
    try:
        grid.knn(q, 10)
        print("mode", mode, "ok", grid.stats()["expand_promotions"], grid.stats()["knn_rounds"])
    except Exception as e:
        print("mode", mode, "FAIL", e)
        try:
            torch.cuda.synchronize()
        except Exception as e2:
            print("torch:", e2)
        sys.exit(1)
    grid.close()
