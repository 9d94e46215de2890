# final-kernel profiling pass + bulk ingest tile A/B at C1/C2/C3
bash tools/profile_c3.sh r2
for r in 1 2; do
for L in paper_conf_icde_li0qhdy18_b200/libggrid.so exp/ing_cpt2.so exp/ing_cpt4.so; do
  echo "lib=$L"
  for c in "1e4 1e7 5 C1" "1e5 1e7 5 C2" "1e6 3.2e7 3 C3"; do
    GGRID_LIB=$PWD/$L GG_INGEST_KERNELS=3 timeout 300 python tools/ingest_probe.py $c 2>&1 | tail -1
  done
done
done
