#!/bin/bash
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/c3_flush_roofline.py --repeat 2 --parity 0 --queries 1024 > gpurun_out/in_c3_$n.log 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/in_c3_$n.log').read().strip().splitlines()[-1]); print('$n C3 ingest %.2f ms %.2f G/s' % (d['ingest_ms'], d['ingest_updates_per_s']/1e9))"
  GG_INGEST_KERNELS=3 GGRID_LIB=$PWD/$L timeout 300 python tools/ingest_probe.py 100000 100000000 3 C2 2>&1 | grep mode= | sed "s/^/$n /" | cut -c1-200
done
