#!/bin/bash
# three-launch ingest (threads, updates per thread) A/B: 1024x8 (default) / 512x16 / 1024x4
for r in 1 2; do
  for v in base t512x16 t1024x4; do
    echo "lib=$v"
    for c in "1e5 1e7 5 C2" "1e6 3.2e7 3 C3"; do
      GGRID_LIB=$PWD/exp/lib_$v.so GG_INGEST_KERNELS=3 timeout 300 python tools/ingest_probe.py $c 2>&1 | tail -1
    done
  done
done
for v in t512x16 t1024x4; do
  GGRID_LIB=$PWD/exp/lib_$v.so timeout 300 python -m pytest tests/test_gpu_ingest.py -m gpu -x -q > gpurun_out/cpt_tests_$v.log 2>&1; echo "$v tests rc=$?"
done
