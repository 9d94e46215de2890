#!/bin/bash
# three-launch ingest tile width A/B (GG_INGEST_CT 256 / 512 / 1024): correctness + large-batch timing
for v in ct256 ct512 ct1024; do
  L=$PWD/exp/lib_$v.so
  GGRID_LIB=$L timeout 300 python -m pytest tests/test_gpu_ingest.py -m gpu -x -q > gpurun_out/ct_tests_$v.log 2>&1; echo "$v tests rc=$?"
  for c in "1e5 1e7 5 C2" "1e4 1e7 5 C1" "1e6 3.2e7 3 C3"; do
    GGRID_LIB=$L GG_INGEST_KERNELS=3 timeout 300 python tools/ingest_probe.py $c 2>&1 | tail -1
  done
done
