#!/bin/bash
# build variant libs: mk.sh name "flags"
set -e
cd /root/repo
d=paper_conf_icpp_jisl0t022_b200/csrc/build/$1; mkdir -p $d
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr -Xptxas -v $2 -c paper_conf_icpp_jisl0t022_b200/csrc/spmspv_flat.cu -o $d/spmspv_flat.o
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/libtsmv.so $d/spmspv_flat.o $(ls paper_conf_icpp_jisl0t022_b200/csrc/build/*.o | grep -v spmspv_flat.o)
