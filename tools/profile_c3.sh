#!/bin/bash
# Round profiling pass at the bench's default workload (C3, one GPU; run under gpurun):
#   1. the launch list of the bench command (gpu__time_duration per launch: cold-cache, serialised)
#   2. ncu --set full of the step's hot kernels: the expansion (first timed step), the flush (the
#      second full flush of the 64M-record log), the three-launch ingest of the 64M bulk batch,
#      and the step's own ingest (k_ingest_direct, 1M updates) and lazy flush (k_flush_warp)
# Usage: tools/profile_c3.sh <tag>; then python tools/summarize_profiles.py <tag>
set -u
TAG=${1:-r2}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
export BENCH_ALLOW_SHORT=1
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-parity --e2e-steps 1"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C3.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-parity --e2e-steps 1 > $OUT/launches_C3.log 2>&1
echo "launch list rc=$?"
cap() {  # name function-name-regex skip
  timeout 1200 ncu --set full --clock-control none --import-source on --kernel-name-base function \
      -k "regex:$2" -s $3 -c 1 -o $OUT/$1 $B > $OUT/$1.log 2>&1
  echo "$1 rc=$?"
}
# the starting expansion level at C3 is the one-warp-per-query kernel (k_expand); the 4th launch
# is the first timed step's
cap expand_C3 '^k_expand$' 3
# flush launches 0-2 are the three full flushes of the 64M-record log (no GC: 2^29-record arena)
cap flush_C3 '^k_flush' 1
cap ingestscatter_C3 '^k_ingest_scatter$' 1
cap ingestclassify_C3 '^k_ingest_classify$' 1
cap stepingest_C3 '^k_ingest_direct$' 3
cap stepflush_C3 '^k_flush_warp$' 3
for f in $OUT/*.ncu-rep; do
  ncu -i $f --page raw --csv > ${f%.ncu-rep}_raw.csv 2>/dev/null
  ncu -i $f --page source --csv > ${f%.ncu-rep}_source.csv 2>/dev/null
done
ls -la $OUT
