#!/bin/bash
# build a variant libtsmv.so with extra nvcc flags for one source file:
#   scripts/mk_variant_file.sh name source.cu "flags"   ->  csrc/build/name/libtsmv.so (TSMV_LIB=...)
set -e
cd /root/repo
d=paper_conf_icpp_jisl0t022_b200/csrc/build/$1; mkdir -p $d
f=$2; o=$(basename $f .cu).o
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr $3 -c paper_conf_icpp_jisl0t022_b200/csrc/$f -o $d/$o
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/libtsmv.so $d/$o $(ls paper_conf_icpp_jisl0t022_b200/csrc/build/*.o | grep -v "/$o")
