#!/bin/bash
export BENCH_ALLOW_SHORT=1
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/pf_b_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/pf_b_$n.log | sed -E 's/kernels.*launch_ms=/ launch_ms=/' | cut -c1-150
  GGRID_LIB=$PWD/$L timeout 600 python tools/c3_flush_roofline.py --repeat 1 --parity 0 > gpurun_out/pf_c3_$n.log 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/pf_c3_$n.log').read().strip().splitlines()[-1]); print('$n C3 knn_qps %.2fM' % (d['knn_qps']/1e6))"
  GGRID_LIB=$PWD/$L timeout 600 python tools/k_sweep.py --k 30,50 --parity 0 --out gpurun_out/pf_c2_$n.jsonl 2>&1 | grep "C2 k=" | sed "s/^/$n /"
done
