#!/bin/bash
mkdir -p gpurun_out
timeout 2400 python -m pytest tests/ -x -q -m gpu > gpurun_out/pytest_full.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_full.log
timeout 900 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 3000 python bench.py --config C5 --steps 5 --warmup 3 --json-out gpurun_out/bench_C5.json > gpurun_out/bench_C5.log 2>&1; echo C5=$?
