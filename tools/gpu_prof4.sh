#!/bin/bash
mkdir -p gpurun_out
timeout 1800 bash tools/profile_round.sh r01; echo prof=$?
timeout 900 python bench.py --config C4 --streams 1 --no-cpu-baseline --json-out gpurun_out/bench_C4_s1.json > gpurun_out/bench_C4_s1.log 2>&1; echo C4s1=$?
