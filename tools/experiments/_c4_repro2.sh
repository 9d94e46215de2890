#!/bin/bash
# the C1 half of the C4 sweep (one process), 2,048-update tile lib then the default, twice
for r in 1 2; do
for L in $PWD/exp/lib_ct256.so ""; do
  echo "lib=${L:-default} pass $r"
  GGRID_LIB=$L timeout 400 python tools/c4_sweep.py --graphs C1 --out gpurun_out/c4_rep2.jsonl > gpurun_out/c4_rep2_tmp.log 2>&1; echo "rc=$?"
  grep "r=\|Error" gpurun_out/c4_rep2_tmp.log | cut -c1-120 | tail -4
done
done
