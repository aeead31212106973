# per-CTA smem now ~2*(8192+896+256+144)=18976 B; 228 KB/SM
for pad in 0 2400 6000 10500 14000; do
  echo "== pad $pad"
  GANNS_DEBUG_SEARCH_SMEM_PAD=$pad python tools/quick_bench.py --l-build 128 --ls 112 --nq-mult 8 --reps 3 2>&1 | grep '"l"'
done
