mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_build.py tests/test_gpu_operating_points.py -x -q > gpurun_out/prof_tests.log 2>&1; tail -1 gpurun_out/prof_tests.log
for c in "C2 128 109" "C3 288 288" "C4 288 288"; do set -- $c
  GANNS_LIB_PATH=ab/libganns_prof.so timeout 900 python tools/phase_breakdown.py --config $1 --l $2 --e $3 2>&1 | tail -1
done | tee gpurun_out/phase_breakdown.log
