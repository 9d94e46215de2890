#!/bin/bash
# r04 measurement pass: profiles, C3 roofline + query batch, C2 k sweep
bash tools/profile_round.sh r04 > gpurun_out/prof_r04.log 2>&1; echo "profile rc=$?"
timeout 900 python tools/c3_flush_roofline.py > gpurun_out/c3_r04.log 2>&1; echo "c3 rc=$?"; tail -1 gpurun_out/c3_r04.log | cut -c1-300
timeout 900 python tools/k_sweep.py --out gpurun_out/k_sweep_C2_r04.jsonl > gpurun_out/k_sweep_C2_r04.log 2>&1; echo "ksweep rc=$?"; tail -8 gpurun_out/k_sweep_C2_r04.log | cut -c1-200
