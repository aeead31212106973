#!/bin/bash
# build-time A/B of libganns_{A,B}.so: C2 build (group sizes), 2 reps each, alternating
for rep in 1 2; do
  for v in A B; do
    echo "== $v rep $rep"
    GANNS_LIB_PATH=$PWD/paper_conf_icde_yuwzqzl22_b200/libganns_$v.so python tools/build_breakdown.py C2 128 ${1:-1024,2048} 2>&1 | grep group
  done
done
