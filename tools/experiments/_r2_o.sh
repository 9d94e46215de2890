python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
GGRID_LIB=$PWD/exp/lib_pair4.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/gputests_pair2.log 2>&1; tail -2 gpurun_out/gputests_pair2.log
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 4 > gpurun_out/var_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/var_$n.log | cut -c1-300
done
GGRID_LIB=$PWD/exp/lib_pair4.so bash tools/ncu_kernel.sh pair_C3 "^k_expand_pair$" 3
