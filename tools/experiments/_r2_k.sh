for rep in 1 2; do
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --config C1 --no-cpu-baseline --e2e-steps 4 > gpurun_out/varC1_$n.log 2>&1
  python tools/bench_summary.py gpurun_out/varC1_$n.log | cut -c1-400
done
done
