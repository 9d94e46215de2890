#!/bin/bash
# r09 measurement pass with the PDL launch chain: profiling pass, then the default bench line twice
bash tools/profile_round.sh r09 > gpurun_out/prof_r09.log 2>&1; echo "profile rc=$?"
timeout 400 python bench.py > gpurun_out/bench_r09b.log 2>&1; echo "bench rc=$?"
timeout 400 python bench.py > gpurun_out/bench_r09c.log 2>&1; echo "bench2 rc=$?"
