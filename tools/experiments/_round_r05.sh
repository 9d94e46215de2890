#!/bin/bash
# r05 measurement pass: the default bench line, the profiling pass, C3
timeout 400 python bench.py > gpurun_out/bench_r05.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_r05.log | cut -c1-400
bash tools/profile_round.sh r05 > gpurun_out/prof_r05.log 2>&1; echo "profile rc=$?"
timeout 900 python tools/c3_flush_roofline.py > gpurun_out/c3_r05.log 2>&1; echo "c3 rc=$?"
