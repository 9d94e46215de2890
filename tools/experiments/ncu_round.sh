#!/bin/bash
# Profiling pass for one round (run under gpurun on ONE GPU):
#   1. launch list of the bench command (gpu__time_duration per launch, cold-cache, serialised)
#   2. ncu --set full of each hot kernel (one launch after warm-up)
# Usage: tools/ncu_round.sh <tag> [bench args...]
set -u
TAG=${1:-r01}; shift || true
ARGS="$@"
OUT=gpurun_out/ncu_$TAG
mkdir -p $OUT
export BENCH_ALLOW_SHORT=1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 $ARGS > $OUT/launches_bench.log 2>&1
echo "launch list rc=$?"
for K in k_expand k_flush k_ingest_classify k_ingest_scatter; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 \
      -o $OUT/full_$K python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 $ARGS > $OUT/full_$K.log 2>&1
  echo "$K rc=$?"
done
ls -la $OUT
