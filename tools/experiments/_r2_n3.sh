python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_prior_art.py -x -q > gpurun_out/gputest_pa_r2e.log 2>&1; tail -3 gpurun_out/gputest_pa_r2e.log
timeout 900 python tools/n3_refine.py --config C1 --queries 2048 > gpurun_out/n3_refine_C1_r2e.log 2>&1; tail -c 1500 gpurun_out/n3_refine_C1_r2e.log
timeout 1200 python tools/n3_refine.py --config C3 --queries 1024 > gpurun_out/n3_refine_C3_r2e.log 2>&1; tail -c 1500 gpurun_out/n3_refine_C3_r2e.log
bash tools/ncu_kernel.sh flushtma_C3 "^k_flush_tma$" 1
