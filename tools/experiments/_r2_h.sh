python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gputests_r2h.log 2>&1; tail -3 gpurun_out/gputests_r2h.log
timeout 600 python bench.py > gpurun_out/bench_C3_r2h.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C3_r2h.log
timeout 600 python bench.py --config C1 --no-cpu-baseline > gpurun_out/bench_C1_r2h.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C1_r2h.log
