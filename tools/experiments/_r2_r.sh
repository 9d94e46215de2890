for rep in 1 2; do
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --no-parity --e2e-steps 1 --steps 3 > gpurun_out/varF_$n.log 2>&1
  python - gpurun_out/varF_$n.log <<'PY'
import json,sys
d=[json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
if not d: print(sys.argv[1], "no line"); sys.exit()
d=d[-1]; f=d["flush"]
print(sys.argv[1], "flush full %.4f ms %.0f GB/s frac %.3f | step flush %.4f ms expand %.4f" % (f["ms"], f["achieved_gbs"], f["frac"], d["per_kernel"]["flush"]["ms_per_step"], d["per_kernel"]["expand"]["ms_per_step"]))
PY
done
done
GGRID_LIB=$PWD/exp/lib_tmw2ts8.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k flush > gpurun_out/gputests_r2r.log 2>&1; tail -2 gpurun_out/gputests_r2r.log
