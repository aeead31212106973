#!/bin/bash
# pipelined (2-stream, back-to-back batches) timing of libganns_{A,B,C}.so in one GPU session
LS=${1:-112,128}
for rep in 1 2; do
  for v in A B C; do
    [ -f paper_conf_icde_yuwzqzl22_b200/libganns_$v.so ] || continue
    echo "== $v rep $rep"
    GANNS_LIB_PATH=$PWD/paper_conf_icde_yuwzqzl22_b200/libganns_$v.so python tools/quick_bench.py --l-build 128 --ls $LS --reps 5 --overlap 8 ${QB_EXTRA:-} 2>&1 | grep '"l"'
  done
done
