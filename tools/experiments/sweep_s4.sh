#!/bin/bash
export BENCH_ALLOW_SHORT=1
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/sw_${n}.log 2>&1
  python tools/bench_summary.py gpurun_out/sw_${n}.log
done
