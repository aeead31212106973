#!/bin/bash
# A/B kernel timing in one GPU session: alternate libganns_A.so / libganns_B.so
LS=${1:-64,112,128}
for rep in 1 2; do
  for v in A B; do
    echo "== $v rep $rep"
    GANNS_LIB_PATH=$PWD/paper_conf_icde_yuwzqzl22_b200/libganns_$v.so python tools/quick_bench.py --l-build 128 --ls $LS --reps 7 2>&1 | grep '"l"'
  done
done
