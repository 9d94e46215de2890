#!/bin/bash
# build experiment variants of libggrid.so into exp/ (flags per variant); edit the list below
cd /root/repo
mkdir -p exp
build() { GGRID_LIB_OUT=exp/lib_$1.so GGRID_NVCC_FLAGS="$2" python -m paper_conf_icde_li0qhdy18_b200.build --force > /dev/null && echo "built $1"; }
build cta2 "" &
build cta1 "-DGG_CTA_LEVEL=1" &
build cta0 "-DGG_CTA_LEVEL=0" &
wait
