#!/bin/bash
# r07 (final) measurement pass: the default bench line, the profiling pass
timeout 400 python bench.py > gpurun_out/bench_r07.log 2>&1; echo "bench rc=$?"
bash tools/profile_round.sh r07 > gpurun_out/prof_r07.log 2>&1; echo "profile rc=$?"
timeout 400 python bench.py > gpurun_out/bench_r07b.log 2>&1; echo "bench2 rc=$?"
