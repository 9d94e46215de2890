#!/bin/bash
# Round profiling pass (one GPU): launch list of the default bench, ncu --set full of the
# expand kernel (C1 bench) and of the flush kernel at USA scale (C3 tool), raw metric dumps.
# Usage: tools/profile_round.sh r01
set -u
TAG=${1:-r01}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
export BENCH_ALLOW_SHORT=1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C1.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $OUT/launches_C1.log 2>&1
echo "launch list rc=$?"
# the starting level's kernel (k_expand_cta<4>) alternates with the chained level's (<8>): the 5th match
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_cta -s 4 -c 1 \
    -o $OUT/expand_C1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $OUT/expand_C1.log 2>&1
echo "expand rc=$?"
# one fused ingest launch per step (batches that fit one resident wave)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ingest -s 3 -c 1 \
    -o $OUT/ingest_C1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $OUT/ingest_C1.log 2>&1
echo "ingest rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_flush -s 1 -c 1 \
    -o $OUT/flush_C3 python tools/c3_flush_roofline.py --parity 0 --queries 1024 --repeat 2 > $OUT/flush_C3.log 2>&1
echo "flush rc=$?"
for f in $OUT/*.ncu-rep; do ncu -i $f --page raw --csv > ${f%.ncu-rep}_raw.csv 2>/dev/null; done
ls -la $OUT
