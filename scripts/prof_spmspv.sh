#!/bin/bash
# ncu evidence for the SpMSpV hot path (run under gpurun from the repo root)
set -x
OUT=${1:-gpurun_out}
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'k_xscan|k_expand|k_compact' -s 6 -c 30 --csv \
    --log-file $OUT/launches.csv python bench.py --steps 8 --warmup 2 --no-bfs --no-cpu > $OUT/ncu_launch_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:'k_xscan|k_expand|k_compact' -s 6 -c 3 \
    -o $OUT/prof_spmspv -f python bench.py --steps 3 --warmup 2 --no-bfs --no-cpu > $OUT/ncu_full.log 2>&1
