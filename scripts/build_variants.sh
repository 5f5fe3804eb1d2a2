#!/bin/bash
# build libtsmv variants of the fused SpMSpV kernel: scripts/build_variants.sh "FB,CB" ...
set -e
cd /root/repo/paper_conf_icpp_jisl0t022_b200/csrc
python ../build.py > /dev/null
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr"
for v in "$@"; do
  IFS=, read FB CB EX <<< "$v"
  d=build/var_${FB}_${CB}${EX//[ =-]/}; mkdir -p $d
  nvcc $F -Xptxas -v -DTSMV_FB=$FB -DTSMV_CB=$CB $EX -c spmspv.cu -o $d/spmspv.o 2> $d/ptxas.log &
done
wait
for v in "$@"; do
  IFS=, read FB CB EX <<< "$v"
  d=build/var_${FB}_${CB}${EX//[ =-]/}
  nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/libtsmv.so $d/spmspv.o $(ls build/*.o | grep -v spmspv.o)
  echo "$v: $(grep -A3 'k_spmspv_fusedILi16EddLi0E' $d/ptxas.log | grep -E 'registers|spill' | tr '\n' ' ')"
done
