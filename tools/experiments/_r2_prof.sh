python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
bash tools/profile_c3.sh r2 > gpurun_out/profile_r2.log 2>&1; tail -3 gpurun_out/profile_r2.log
timeout 600 python bench.py > gpurun_out/bench_C3_r2m.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C3_r2m.log
