python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gputests_r2u.log 2>&1; tail -3 gpurun_out/gputests_r2u.log
for rep in 1 2; do
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 4 > gpurun_out/var_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/var_$n.log | cut -c1-330
done
done
timeout 600 python bench.py --config C1 --no-cpu-baseline > gpurun_out/bench_C1_r2u.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C1_r2u.log | cut -c1-330
