#!/bin/bash
export BENCH_ALLOW_SHORT=1
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/sw_b_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/sw_b_$n.log | cut -c1-260
  GGRID_LIB=$PWD/$L timeout 600 python tools/c3_flush_roofline.py --repeat 3 --parity 0 > gpurun_out/sw_c3_$n.log 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/sw_c3_$n.log').read().strip().splitlines()[-1]); print('$n C3 flush %.3f ms %.0f GB/s knn %.2fM' % (d['flush_ms'], d['flush_gbs'], d['knn_qps']/1e6))"
done
