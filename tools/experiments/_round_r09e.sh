#!/bin/bash
# r09: C4 update-heavy sweep and C3 (flush roofline + sampled parity) with the 8,192-update ingest tiles
timeout 900 python tools/c4_sweep.py --out gpurun_out/c4_sweep_r09.jsonl > gpurun_out/c4_sweep_r09.log 2>&1; echo "c4 rc=$?"
timeout 900 python tools/c3_flush_roofline.py > gpurun_out/c3_r09.log 2>&1; echo "c3 rc=$?"
