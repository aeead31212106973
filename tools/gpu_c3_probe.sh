# C3 wide-form probe: parity of every rows-per-round, a full ncu capture at the
# bench operating point, 1-warp CTAs, and the C5 bench line on small shards.
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "wide_rows or shapes" > gpurun_out/t3_wide.log 2>&1; echo wide=$?
for v in default W1; do
  if [ $v = W1 ]; then export GANNS_LIB_PATH=$PWD/paper_conf_icde_yuwzqzl22_b200/libganns_W1.so; fi
  for wr in auto 4 2; do
    if [ $wr = auto ]; then unset GANNS_WIDE_ROWS; else export GANNS_WIDE_ROWS=$wr; fi
    echo "== $v wide rows $wr"; python tools/quick_bench.py --config C3 --l-build 128 --ls 320 --reps 5 2>&1 | grep '"l"'
  done
done > gpurun_out/c3_probe.log 2>&1
unset GANNS_LIB_PATH GANNS_WIDE_ROWS
ncu --set full --clock-control none --import-source on -k regex:^search_kernel -s 2 -c 1 \
    -o gpurun_out/c3_full python tools/prof_search.py --config C3 --l 320 --e 320 --l-build 128 > gpurun_out/c3_ncu.log 2>&1
python tools/ncu_summary.py gpurun_out/c3_full.ncu-rep > gpurun_out/c3_ncu_summary.json 2>&1
python tools/ncu_lines.py gpurun_out/c3_full.ncu-rep > gpurun_out/c3_ncu_lines.txt 2>&1
timeout 1200 python bench.py --config C5 --shard-rows 500000 --steps 3 --warmup 3 --cpu-seconds 5 > gpurun_out/c5_small.log 2>&1; echo c5=$?
