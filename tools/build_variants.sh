#!/bin/bash
# build experiment variants of libggrid.so into exp/ (flags per variant); edit the list below
cd /root/repo
build() { GGRID_LIB_OUT=exp/lib_$1.so GGRID_NVCC_FLAGS="$2" python -m paper_conf_icde_li0qhdy18_b200.build --force > /dev/null && echo "built $1"; }
build base "" &
build h512 "-DGG_H0=512 -DGG_F0=128" &
build f128 "-DGG_F0=128" &
build h2048 "-DGG_H0=2048" &
wait
