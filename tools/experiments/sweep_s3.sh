#!/bin/bash
# H0 x delta sweep of the level-0 expansion (experiment variants in exp/)
export BENCH_ALLOW_SHORT=1
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  for d in ${DELTAS:-0 1500 2000}; do
    GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 --delta $d > gpurun_out/sw_${n}_d$d.log 2>&1
    python tools/bench_summary.py gpurun_out/sw_${n}_d$d.log
  done
done
