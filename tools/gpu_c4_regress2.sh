timeout 1200 python -m pytest tests/test_gpu_sanitizer.py -q > gpurun_out/t8_san.log 2>&1; echo san=$?
for v in old new; do
  if [ $v = old ]; then export GANNS_LIB_PATH=$PWD/paper_conf_icde_yuwzqzl22_b200/libganns_old.so; else unset GANNS_LIB_PATH; fi
  echo "== $v"; timeout 900 python bench.py --config C4 --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-300
done > gpurun_out/c4_regress2.log 2>&1
