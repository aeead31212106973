set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/t2_parity.log 2>&1; echo parity=$?
bash tools/ab_bench.sh 112,128 > gpurun_out/ab_pf.log 2>&1
for wr in 8 auto 6 4; do
  if [ $wr = auto ]; then unset GANNS_WIDE_ROWS; else export GANNS_WIDE_ROWS=$wr; fi
  echo "== wide rows $wr"; python tools/quick_bench.py --config C3 --l-build 128 --ls 160,320 --reps 5 2>&1 | grep '"l"'
done > gpurun_out/c3_wrows.log 2>&1
