#!/bin/bash
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 600 python tools/c3_flush_roofline.py --repeat 4 --parity 0 > gpurun_out/pd_c3_$n.log 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/pd_c3_$n.log').read().strip().splitlines()[-1]); print('$n C3 flush %.3f ms %.0f GB/s (%.1f%%) best %.0f' % (d['flush_ms'], d['flush_gbs'], 100*d['flush_frac_of_peak'], d['flush_best_gbs']))"
done
