#!/bin/bash
# ncu --set full of the C3 step's ingest (k_ingest_direct) and warp-per-cell flush (k_flush_warp),
# one launch each from the first timed step.  Usage (under gpurun): bash tools/ncu_two.sh <tag>
TAG=${1:-x}
OUT=gpurun_out/ncu
mkdir -p $OUT
export BENCH_ALLOW_SHORT=1
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-parity --e2e-steps 1"
for spec in "ingestdirect:^k_ingest_direct$:3" "flushwarp:^k_flush_warp$:3"; do
  IFS=: read NAME K S <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
      -k "regex:$K" -s $S -c 1 -o $OUT/${NAME}_$TAG $B > $OUT/${NAME}_$TAG.log 2>&1
  echo "$NAME rc=$?"
  ncu -i $OUT/${NAME}_$TAG.ncu-rep --page raw --csv > $OUT/${NAME}_${TAG}_raw.csv 2>/dev/null
done
