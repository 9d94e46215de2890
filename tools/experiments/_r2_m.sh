# three-launch ingest tile size A/B (step batch fills 123 of 148 SMs at 8,192-update tiles)
for r in 1 2; do
for L in paper_conf_icde_li0qhdy18_b200/libggrid.so exp/ing_*.so; do
  n=$(basename $L .so)
  for c in C3 C1; do
    GGRID_LIB=$PWD/$L timeout 300 python bench.py --config $c --no-cpu-baseline --no-parity --e2e-steps 1 --steps 3 > gpurun_out/varI_${n}_$c.log 2>&1
    python - gpurun_out/varI_${n}_$c.log <<'PY'
import json,sys
d=[json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
if not d: print(sys.argv[1], "no line"); sys.exit()
d=d[-1]; pk=d["per_kernel"]
print(sys.argv[1], "qps %.2fM ms/step %.4f ingest %.4f flush %.4f expand %.4f" % (d["value"]/1e6, d["ms_per_step"], pk["ingest"]["ms_per_step"], pk["flush"]["ms_per_step"], pk["expand"]["ms_per_step"]))
PY
  done
  GGRID_LIB=$PWD/$L GG_INGEST_KERNELS=3 timeout 300 python tools/ingest_probe.py 1e6 3.2e7 3 C3 2>&1 | tail -1
done
done
for L in exp/ing_*.so; do
  GGRID_LIB=$PWD/$L timeout 300 python -m pytest tests/test_gpu_ingest.py -m gpu -x -q > gpurun_out/ing_tests_$(basename $L .so).log 2>&1; echo "$L tests rc=$?"
done
