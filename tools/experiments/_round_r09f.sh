#!/bin/bash
# r09 final: GPU suite, the C1 C4 sweep looped with GGRID_DEBUG=1 (rejection diagnosis), bench line
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_r09f.log 2>&1; echo "tests rc=$?"
for r in 1 2 3; do
  GGRID_DEBUG=1 timeout 400 python tools/c4_sweep.py --graphs C1 --out gpurun_out/c4_loop.jsonl > gpurun_out/c4_loop_$r.log 2>&1; echo "sweep $r rc=$?"
  grep "ggrid_ingest\|Error" gpurun_out/c4_loop_$r.log | head -5
done
timeout 400 python bench.py > gpurun_out/bench_r09f.log 2>&1; echo "bench rc=$?"
