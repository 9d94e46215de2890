#!/bin/bash
export BENCH_ALLOW_SHORT=1
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/c4_sweep.py --graphs C2 --objects 1e4 --r 10 --out gpurun_out/bf_$n.jsonl 2>&1 | grep "r=" | sed "s/^/$n /" | cut -c1-150
  GGRID_LIB=$PWD/$L timeout 600 python tools/c4_sweep.py --graphs C1 --objects 1e4 --r 10 --out gpurun_out/bf1_$n.jsonl 2>&1 | grep "r=" | sed "s/^/$n /" | cut -c1-150
done
