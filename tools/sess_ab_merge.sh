mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_build.py tests/test_gpu_hnsw.py tests/test_gpu_operating_points.py tests/test_gpu_dist_build.py tests/test_gpu_knn.py -x -q > gpurun_out/ab2_tests.log 2>&1; tail -2 gpurun_out/ab2_tests.log
for lib in paper_conf_icde_yuwzqzl22_b200/libganns.so ab/libganns_base.so; do
  echo "== $lib"; GANNS_LIB_PATH=$lib timeout 600 python tools/build_phases.py 4 2>&1 | grep rep | tail -2
  GANNS_LIB_PATH=$lib timeout 600 python tools/search_ab.py --config C2 --l 128 --e 109 2>&1 | tail -1
done | tee gpurun_out/ab2_merge.log
