#!/bin/bash
# locality order A/B: GANNS_ORDER = pivots (0 = off), pipelined quick bench, 2 reps
for rep in 1 2; do
  for P in 0 16 64; do
    echo "== P=$P rep $rep"
    GANNS_ORDER=$P python tools/quick_bench.py --l-build 128 --ls 112,128 --reps 5 --overlap 8 2>&1 | grep '"streams": 2'
  done
done
