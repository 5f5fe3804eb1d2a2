#!/bin/bash
# build a variant libtsmv.so replacing one object with another source file:
#   scripts/mk_variant_src.sh name path/to/variant.cu object.o "flags"
set -e
cd /root/repo
d=paper_conf_icpp_jisl0t022_b200/csrc/build/$1; mkdir -p $d
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr \
     -I paper_conf_icpp_jisl0t022_b200/csrc $4 -c $2 -o $d/$3
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/libtsmv.so $d/$3 $(ls paper_conf_icpp_jisl0t022_b200/csrc/build/*.o | grep -v "/$3")
