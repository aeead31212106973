#!/bin/bash
mkdir -p gpurun_out
bash tools/ab_bench.sh 96,112 > gpurun_out/ab2.log 2>&1; echo ab=$?
python tools/quick_bench.py --l-build 128 --ls 112 --reps 7 --orders 16,64,256,1024 --nq-mult 1,4 > gpurun_out/order.log 2>&1; echo order=$?
timeout 900 python -m pytest tests/test_gpu_sanitizer.py tests/test_gpu_parity.py tests/test_gpu_build.py -x -q > gpurun_out/pytest_ab2.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_ab2.log
