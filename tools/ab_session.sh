#!/bin/bash
# GPU A/B session: parity of the default library on the build/search tests, then
# A/B of the variants in ab/ (tools/build_variants.sh).  Results: gpurun_out/ab_*.log
mkdir -p gpurun_out
D=paper_conf_icde_yuwzqzl22_b200/libganns.so
timeout 1200 python -m pytest tests/test_gpu_build.py tests/test_gpu_dist_build.py tests/test_gpu_parity.py tests/test_gpu_hnsw.py -x -q > gpurun_out/ab_tests.log 2>&1
tail -2 gpurun_out/ab_tests.log
for lib in $D ab/libganns_p0.so $D ab/libganns_p0.so; do
  GANNS_LIB_PATH=$lib timeout 600 python tools/build_once.py C2 5 2>&1 | tail -1
done | tee gpurun_out/ab_build.log
for lib in $D ab/libganns_nohint.so; do
  GANNS_LIB_PATH=$lib timeout 900 python tools/search_ab.py --config C3 --l 288 2>&1 | tail -1
done | tee gpurun_out/ab_c3_hint.log
for lib in $D ab/libganns_noinline.so; do
  GANNS_LIB_PATH=$lib timeout 900 python tools/search_ab.py --config C4 --l 288 2>&1 | tail -1
done | tee gpurun_out/ab_c4_noinline.log
for solo in 1 0; do
  GANNS_SOLO=$solo timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --json-out gpurun_out/ab_solo$solo.json > /dev/null 2>&1
  python -c "import json; d=json.load(open('gpurun_out/ab_solo$solo.json')); print('solo $solo', d['value'], d['config']['strong_scaling_proxy'])"
done | tee gpurun_out/ab_solo.log
