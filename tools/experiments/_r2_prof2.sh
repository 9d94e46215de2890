python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
bash tools/profile_c3.sh r2 > gpurun_out/profile_r2.log 2>&1; tail -2 gpurun_out/profile_r2.log
timeout 600 python bench.py --config C1 --no-cpu-baseline > gpurun_out/bench_C1_r2t.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C1_r2t.log
timeout 900 python tools/n3_refine.py --config C3 --queries 2048 > gpurun_out/n3_refine_C3_r2t.log 2>&1; tail -c 600 gpurun_out/n3_refine_C3_r2t.log
