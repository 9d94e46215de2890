#!/bin/bash
# tile 8,192 (GG_INGEST_CT=1024, new default) vs 2,048 (exp/lib_ct256.so): full GPU suite, then
# same-box large-batch three-launch ingest A/B, alternating, twice
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_r09d.log 2>&1; echo "tests rc=$?"
for r in 1 2; do
  for L in "" $PWD/exp/lib_ct256.so; do
    echo "lib=${L:-default}"
    for c in "1e5 1e7 5 C2" "1e4 1e7 5 C1" "1e6 3.2e7 3 C3"; do
      GGRID_LIB=$L GG_INGEST_KERNELS=3 timeout 300 python tools/ingest_probe.py $c 2>&1 | tail -1
    done
  done
done
timeout 400 python bench.py > gpurun_out/bench_r09d.log 2>&1; echo "bench rc=$?"
