python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_prior_art.py tests/test_gpu_ingest.py -x -q > gpurun_out/gputests_r2f.log 2>&1; tail -3 gpurun_out/gputests_r2f.log
for L in exp/lib_*.so; do
  n=$(basename $L .so)
  GGRID_LIB=$PWD/$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/var_$n.log 2>&1
  python - gpurun_out/var_$n.log <<'PY'
import json,sys
d=[json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
if not d: print(sys.argv[1], "no line"); sys.exit()
d=d[-1]; f=d["flush"]
print(sys.argv[1], "qps %.2fM flush full %.4f ms %.0f GB/s frac %.3f | step flush %.4f ms expand %.4f promo %.1f parity %s" % (d["value"]/1e6, f["ms"], f["achieved_gbs"], f["frac"], d["per_kernel"]["flush"]["ms_per_step"], d["per_kernel"]["expand"]["ms_per_step"], d["expand_promotions_per_step"], d["parity"]["rows_exact"]))
PY
done
timeout 900 python tools/n3_refine.py --config C1 --queries 2048 > gpurun_out/n3_refine_C1_r2f.log 2>&1; tail -c 900 gpurun_out/n3_refine_C1_r2f.log
timeout 1200 python tools/n3_refine.py --config C3 --queries 2048 > gpurun_out/n3_refine_C3_r2f.log 2>&1; tail -c 900 gpurun_out/n3_refine_C3_r2f.log
