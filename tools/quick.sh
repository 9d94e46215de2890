#!/bin/bash
# Quick GPU check of a kernel change: GPU parity tests + one bench line (summary).
# Usage (under gpurun): bash tools/quick.sh [tag] [bench args...]
TAG=${1:-q}; shift || true
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/quick_$TAG.tests.log 2>&1
echo "tests rc=$? $(tail -1 gpurun_out/quick_$TAG.tests.log)"
BENCH_ALLOW_SHORT=1 timeout 400 python bench.py --no-cpu-baseline --e2e-steps 3 "$@" > gpurun_out/quick_$TAG.bench.log 2>&1
echo "bench rc=$?"
tail -1 gpurun_out/quick_$TAG.bench.log | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('qps %.2fM  ms/step %.4f  expand launch ms %.4f  e2e %.2fM  clocks %s' % (d['value']/1e6, d['ms_per_step'], d['roofline']['launch_ms'], d['e2e']['value']/1e6, d['clocks']['sm_mhz']))
print({k: (round(v['ms_per_step'],4) if isinstance(v, dict) else v) for k, v in d['per_kernel'].items()})
print(d['expand_work_per_query'], d['knn_rounds_per_step'])"
