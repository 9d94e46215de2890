#!/bin/bash
# r09 re-entry validation: GPU tests, smoke, default bench line
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_r09.log 2>&1; echo "tests rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_r09.log 2>&1; echo "smoke rc=$?"
timeout 400 python bench.py > gpurun_out/bench_r09.log 2>&1; echo "bench rc=$?"
