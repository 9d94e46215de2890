#!/bin/bash
# alternating A/B bench runs of the experiment libraries in exp/
export BENCH_ALLOW_SHORT=1
for i in 1 2 3; do
  for L in exp/lib_*.so; do
    n=$(basename $L .so)
    GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 6 > gpurun_out/ab_${n}_$i.log 2>&1
    python tools/bench_summary.py gpurun_out/ab_${n}_$i.log | sed -E "s/kernels.*launch_ms=/ launch_ms=/" | cut -c1-140
  done
done
