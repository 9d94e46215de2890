#!/bin/bash
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/k_sweep.py --k 40,50,100,200 --parity 0 --out gpurun_out/wl_c2_$n.jsonl > gpurun_out/wl_c2_$n.log 2>&1
  grep "C2 k=" gpurun_out/wl_c2_$n.log | sed "s/^/$n /"
done
