#!/bin/bash
# A/B/C (libganns_{A,B,C}.so) on C2, then the GPU parity suite on the current libganns.so
mkdir -p gpurun_out
bash tools/abc_bench.sh ${1:-96,112} > gpurun_out/abc.log 2>&1; echo abc=$?
timeout 1200 python -m pytest ${PYTEST_FILES:-tests/test_gpu_sanitizer.py tests/test_gpu_parity.py tests/test_gpu_build.py} -x -q > gpurun_out/pytest_abc.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_abc.log
