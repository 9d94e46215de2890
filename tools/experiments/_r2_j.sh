python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
for rep in 1 2; do
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 4 > gpurun_out/var_base.log 2>&1; python tools/bench_summary.py gpurun_out/var_base.log | cut -c1-300
GGRID_SORT_QUERIES=1 timeout 300 python bench.py --no-cpu-baseline --e2e-steps 4 > gpurun_out/var_sortq.log 2>&1; python tools/bench_summary.py gpurun_out/var_sortq.log | cut -c1-300
done
bash tools/ncu_kernel.sh flushtma2_C3 "^k_flush_tma$" 1
