#!/bin/bash
# ncu --set full of one kernel (regex $1) in a short bench run; extra args go to bench.py
K=$1; TAG=$2; shift 2
mkdir -p gpurun_out/ncu_$TAG
export BENCH_ALLOW_SHORT=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 \
  -o gpurun_out/ncu_$TAG/full_$K python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 "$@" \
  > gpurun_out/ncu_$TAG/full_$K.log 2>&1
echo "$K rc=$?"
