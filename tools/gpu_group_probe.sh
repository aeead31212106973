# Warp-group wide form: parity, C3 timing group vs one-warp, ncu capture.
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "wide_rows or shapes" > gpurun_out/t4_group.log 2>&1; echo parity=$?
for grp in 1 0; do
  export GANNS_WIDE_GROUP=$grp
  for wr in auto 4 8; do
    if [ $wr = auto ]; then unset GANNS_WIDE_ROWS; else export GANNS_WIDE_ROWS=$wr; fi
    echo "== group $grp wide rows $wr"; python tools/quick_bench.py --config C3 --l-build 128 --ls 160,320 --reps 5 2>&1 | grep '"l"'
  done
done > gpurun_out/c3_group.log 2>&1
unset GANNS_WIDE_GROUP GANNS_WIDE_ROWS
ncu --set full --clock-control none --import-source on -k regex:^search_group -s 2 -c 1 \
    -o gpurun_out/c3g_full python tools/prof_search.py --config C3 --l 320 --e 320 --l-build 128 > gpurun_out/c3g_ncu.log 2>&1
python tools/ncu_summary.py gpurun_out/c3g_full.ncu-rep > gpurun_out/c3g_ncu_summary.json 2>&1
python tools/ncu_lines.py gpurun_out/c3g_full.ncu-rep > gpurun_out/c3g_ncu_lines.txt 2>&1
