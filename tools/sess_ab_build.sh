# build A/B on the GPU clock: default library vs ab/libganns_base.so, + parity of the default
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_build.py tests/test_gpu_operating_points.py tests/test_gpu_dist_build.py tests/test_gpu_hnsw.py -x -q > gpurun_out/ab3_tests.log 2>&1; tail -1 gpurun_out/ab3_tests.log
for lib in paper_conf_icde_yuwzqzl22_b200/libganns.so ab/libganns_base.so paper_conf_icde_yuwzqzl22_b200/libganns.so; do
  echo "== $lib"; GANNS_LIB_PATH=$lib timeout 600 python tools/build_phases.py 3 2>&1 | grep rep | tail -1
done | tee gpurun_out/ab3_build.log
