#!/bin/bash
# build a variant lib with bfs_fused.cu compiled under extra flags: mk_variant_bfs.sh name "flags"
set -e
cd /root/repo
d=paper_conf_icpp_jisl0t022_b200/csrc/build/$1; mkdir -p $d
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr -Xptxas -v $2 -c paper_conf_icpp_jisl0t022_b200/csrc/bfs_fused.cu -o $d/bfs_fused.o 2>&1 | grep -A1 "k_bfs_fusedILi16" | tail -1
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/libtsmv.so $d/bfs_fused.o $(ls paper_conf_icpp_jisl0t022_b200/csrc/build/*.o | grep -v bfs_fused.o)
