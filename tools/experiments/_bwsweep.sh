#!/bin/bash
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/c4_sweep.py --graphs C2 --objects 1e4 --r 10 --out gpurun_out/bw_$n.jsonl 2>&1 | grep "r=" | sed "s/^/$n /" | cut -c1-150
  GGRID_LIB=$PWD/$L timeout 600 python tools/k_sweep.py --k 100,200 --parity 0 --out gpurun_out/bwk_$n.jsonl 2>&1 | grep "C2 k=" | sed "s/^/$n /"
done
