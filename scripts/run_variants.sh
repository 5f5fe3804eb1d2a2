#!/bin/bash
# run scripts/sweep.py for each built variant directory given
for v in "$@"; do
  echo "== $v"
  TSMV_LIB=paper_conf_icpp_jisl0t022_b200/csrc/build/$v/libtsmv.so timeout 300 python scripts/sweep.py 22 2 0.0001,0.01,0.1 2>&1 | grep thr
  TSMV_LIB=paper_conf_icpp_jisl0t022_b200/csrc/build/$v/libtsmv.so timeout 300 python scripts/sweep.py 14 2 0.1 2>&1 | grep thr
done
