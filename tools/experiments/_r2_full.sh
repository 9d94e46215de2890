python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/gputests_r2c.log 2>&1; tail -15 gpurun_out/gputests_r2c.log
BENCH_DIST_BACKEND=gloo timeout 600 python bench.py --gpus 2 --config C1 --steps 3 --e2e-steps 2 > gpurun_out/bench_gloo2_C1_r2c.log 2>&1; tail -c 1500 gpurun_out/bench_gloo2_C1_r2c.log
timeout 600 python bench.py > gpurun_out/bench_C3_r2c.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C3_r2c.log
