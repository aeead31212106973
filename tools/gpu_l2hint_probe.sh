# L2 residency hints on C2: evict_last for the vector rows of low-id (early
# inserted hub) vertices, optional evict_first for the rest.
for rep in 1 2; do
for cfg in "0 0" "65536 0" "131072 0" "262144 0" "131072 1" "0 0"; do
  set -- $cfg
  export GANNS_L2_HOT_ROWS=$1 GANNS_L2_COLD_FIRST=$2
  echo "== hot $1 cold_first $2"; python tools/quick_bench.py --l-build 128 --ls 112,128 --reps 7 2>&1 | grep '"l"'
done
done > gpurun_out/l2hint.log 2>&1
