#!/bin/bash
# build experiment variants of libggrid.so into exp/ (flags per variant)
cd /root/repo
build() { GGRID_LIB_OUT=exp/lib_$1.so GGRID_NVCC_FLAGS="$2" python -m paper_conf_icde_li0qhdy18_b200.build --force > /dev/null && echo "built $1"; }
build h0 "-DGG_HASH=0" &
build h1 "-DGG_HASH=1" &
build h2 "-DGG_HASH=2" &
build h0big "-DGG_HASH=0 -DGG_H0=2048" &
build h1big "-DGG_HASH=1 -DGG_H0=2048" &
wait
