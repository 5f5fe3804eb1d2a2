#!/bin/bash
# A/B of flat-kernel build variants (scripts/mk_variant.sh) with scripts/ab.py
cd /root/repo
for v in base v768_77 v768_78 v768_88 v512_88 v1024_78; do
  if [ $v = base ]; then L=paper_conf_icpp_jisl0t022_b200/libtsmv.so; else L=paper_conf_icpp_jisl0t022_b200/csrc/build/$v/libtsmv.so; fi
  echo "== $v"; TSMV_LIB=$L timeout 300 python scripts/ab.py 22 0.0001,0.01,0.1 2>&1 | tail -3
done
