#!/bin/bash
export BENCH_ALLOW_SHORT=1
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/k_sweep.py --k 10,30,40,50 --parity 0 --out gpurun_out/c0_c2_$n.jsonl > gpurun_out/c0_c2_$n.log 2>&1
  grep "C2 k=" gpurun_out/c0_c2_$n.log | sed "s/^/$n /"
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/c0_b_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/c0_b_$n.log | cut -c1-120
done
