#!/bin/bash
# C4 C1 |O|=1e6 r=1000 (1e7-update three-launch batches): new default lib vs the 2,048-update tile lib
for L in "" $PWD/exp/lib_ct256.so; do
  echo "lib=${L:-default}"
  GGRID_LIB=$L timeout 300 python tools/c4_sweep.py --graphs C1 --objects 1e6 --r 1000,10000 --out gpurun_out/c4_repro.jsonl 2>&1 | tail -3 | cut -c1-200
  GGRID_LIB=$L GG_INGEST_KERNELS=3 timeout 300 python tools/ingest_probe.py 1e6 1e7 3 C1 2>&1 | tail -1 | cut -c1-200
done
