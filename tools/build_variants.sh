#!/bin/bash
# build experiment variants of libggrid.so into exp/ (flags per variant):
#   tools/build_variants.sh name1 "flags1" name2 "flags2" ...
cd /root/repo
mkdir -p exp
rm -f exp/lib_*.so
build() { GGRID_LIB_OUT=exp/lib_$1.so GGRID_NVCC_FLAGS="$2" python -m paper_conf_icde_li0qhdy18_b200.build --force > /dev/null && echo "built $1"; }
while [ $# -ge 2 ]; do build "$1" "$2" & shift 2; done
wait
