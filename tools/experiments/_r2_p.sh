python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_configs.py -x -q > gpurun_out/gputests_r2p.log 2>&1; tail -2 gpurun_out/gputests_r2p.log
for rep in 1 2; do
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 4 > gpurun_out/var_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/var_$n.log | cut -c1-300
done
done
