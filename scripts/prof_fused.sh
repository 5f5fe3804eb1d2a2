#!/bin/bash
# ncu full capture of the fused SpMSpV kernel on config T (R-MAT s22, 1 %, fp64)
OUT=${1:-gpurun_out}
mkdir -p $OUT
ncu --set full --clock-control none --import-source on -k regex:k_spmspv_fused -s 5 -c 1 \
    -o $OUT/prof_fused -f python scripts/sweep.py 22 2 0.01 > $OUT/ncu_fused.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:'k_spmspv_fused' -s 3 -c 8 --csv --log-file $OUT/launches_fused.csv python scripts/sweep.py 22 2 0.01 > /dev/null 2>&1
