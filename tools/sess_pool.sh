mkdir -p gpurun_out
timeout 600 python tools/build_phases.py 8 2>&1 | grep rep > gpurun_out/build_phases3.log; cat gpurun_out/build_phases3.log
python tools/build_once.py C2 6 2>&1 | tail -7
timeout 1200 python -m pytest tests/test_gpu_build.py tests/test_gpu_dist_build.py tests/test_gpu_hnsw.py tests/test_gpu_operating_points.py -x -q 2>&1 | tail -2
