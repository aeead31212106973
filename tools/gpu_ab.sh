#!/bin/bash
# A/B (libganns_A.so vs libganns_B.so) on C2, then the GPU parity suite on the current libganns.so
mkdir -p gpurun_out
bash tools/ab_bench.sh ${1:-96,112,128} > gpurun_out/ab.log 2>&1; echo ab=$?
timeout 1500 python -m pytest tests/ -x -q -m gpu ${PYTEST_ARGS:-} > gpurun_out/pytest_ab.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_ab.log
