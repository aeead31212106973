timeout 1200 python -m pytest tests/test_gpu_sanitizer.py -x -q > gpurun_out/t7_san.log 2>&1; echo san=$?
for v in old new old new; do
  if [ $v = old ]; then export GANNS_LIB_PATH=$PWD/paper_conf_icde_yuwzqzl22_b200/libganns_old.so; else unset GANNS_LIB_PATH; fi
  echo "== $v"; python tools/quick_bench.py --config C4 --l-build 128 --ls 128,320 --reps 5 2>&1 | grep '"l"\|build_s'
done > gpurun_out/c4_regress.log 2>&1
unset GANNS_LIB_PATH
bash tools/ab_bench.sh 112,128 > gpurun_out/ab_pair.log 2>&1
