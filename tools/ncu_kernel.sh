#!/bin/bash
# ncu --set full (with source) of one kernel launch of the default bench run (C3).
# Usage: tools/ncu_kernel.sh <out-name> <function-name-regex> <launches-to-skip> [bench args...]
#   e.g. tools/ncu_kernel.sh expand_C3 '^k_expand$' 3
set -u
NAME=$1; K=$2; S=$3; shift 3
OUT=gpurun_out/ncu
mkdir -p $OUT
export BENCH_ALLOW_SHORT=1
timeout 1500 ncu --set full --clock-control none --import-source on --kernel-name-base function \
    -k "regex:$K" -s $S -c 1 -o $OUT/$NAME \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-parity --e2e-steps 1 "$@" > $OUT/$NAME.log 2>&1
echo "$NAME rc=$?"
ncu -i $OUT/$NAME.ncu-rep --page raw --csv > $OUT/${NAME}_raw.csv 2>/dev/null
ncu -i $OUT/$NAME.ncu-rep --page source --csv > $OUT/${NAME}_source.csv 2>/dev/null
ncu -i $OUT/$NAME.ncu-rep --page details --csv > $OUT/${NAME}_details.csv 2>/dev/null
