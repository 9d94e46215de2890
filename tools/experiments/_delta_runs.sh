python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_multi.py -x -q > gpurun_out/gputest_multi_r2a.log 2>&1; tail -3 gpurun_out/gputest_multi_r2a.log
for D in 1545 2060 3090; do
  GGRID_LIB=$PWD/exp/lib_pfh768.so timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 --delta $D > gpurun_out/var_delta$D.log 2>&1
  python tools/bench_summary.py gpurun_out/var_delta$D.log
done
