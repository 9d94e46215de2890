#!/bin/bash
# build experiment variants of libggrid.so into exp/ (flags per variant); edit the list below
cd /root/repo
mkdir -p exp
build() { GGRID_LIB_OUT=exp/lib_$1.so GGRID_NVCC_FLAGS="$2" python -m paper_conf_icde_li0qhdy18_b200.build --force > /dev/null && echo "built $1"; }
build h1024 "" &
build h768 "-DGG_H0=768" &
build h640 "-DGG_H0=640" &
build h896 "-DGG_H0=896" &
wait
