#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_b3.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_b3.log
timeout 900 python bench.py --json-out gpurun_out/bench_C2.json > gpurun_out/bench_C2.log 2>&1; echo C2=$?
for c in C3 C4; do
  timeout 1500 python bench.py --config $c --json-out gpurun_out/bench_$c.json > gpurun_out/bench_$c.log 2>&1; echo $c=$?
done
