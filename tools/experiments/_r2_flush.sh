python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 900 compute-sanitizer --tool memcheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -x -q -k "flush_parity or flush_long or flush_spill or flush_histogram" > gpurun_out/sanitize_flush.log 2>&1; tail -4 gpurun_out/sanitize_flush.log
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ingest.py tests/test_gpu_configs.py -x -q > gpurun_out/gputests_r2d.log 2>&1; tail -3 gpurun_out/gputests_r2d.log
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/var_$n.log 2>&1
  python - gpurun_out/var_$n.log <<'PY'
import json,sys
d=[json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
if not d: print(sys.argv[1], "no line"); sys.exit()
d=d[-1]; f=d["flush"]
print(sys.argv[1], "qps %.2fM flush full %.4f ms %.0f GB/s frac %.3f | step flush %.4f ms expand %.4f parity %s" % (d["value"]/1e6, f["ms"], f["achieved_gbs"], f["frac"], d["per_kernel"]["flush"]["ms_per_step"], d["per_kernel"]["expand"]["ms_per_step"], d["parity"]["rows_exact"]))
PY
done
