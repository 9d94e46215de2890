#!/bin/bash
# A/B of experiment builds in exp/ (tools/build_variants.sh), interleaved R times so box drift
# hits every variant alike: tools/ab.sh <rounds> [bench args]; one summary line per run
R=${1:-2}; shift || true
export BENCH_ALLOW_SHORT=1
for r in $(seq 1 $R); do
  for L in exp/lib_*.so; do
    n=$(basename $L .so)
    GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 --steps 30 "$@" > gpurun_out/ab_${n}_$r.log 2>&1
    echo "$n r$r: $(python tools/bench_summary.py gpurun_out/ab_${n}_$r.log | cut -c1-260)"
  done
done
