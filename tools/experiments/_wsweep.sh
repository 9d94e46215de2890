#!/bin/bash
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/c3_flush_roofline.py --repeat 1 --parity 0 > gpurun_out/ws_c3_$n.log 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/ws_c3_$n.log').read().strip().splitlines()[-1]); print('$n C3 knn_qps %.2fM knn_ms %.3f' % (d['knn_qps']/1e6, d['knn_ms']))"
  GGRID_LIB=$PWD/$L timeout 600 python tools/k_sweep.py --k 10,30 --parity 0 --out gpurun_out/ws_c2_$n.jsonl > gpurun_out/ws_c2_$n.log 2>&1
  grep "C2 k=" gpurun_out/ws_c2_$n.log | sed "s/^/$n /"
done
