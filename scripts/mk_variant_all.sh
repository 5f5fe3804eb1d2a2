#!/bin/bash
# full variant build: /tmp/mkvar.sh name "flags"
set -e
cd /root/repo
d=paper_conf_icpp_jisl0t022_b200/csrc/build/$1; mkdir -p $d
for f in paper_conf_icpp_jisl0t022_b200/csrc/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr $2 -c $f -o $d/$(basename $f .cu).o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/libtsmv.so $d/*.o
