#!/bin/bash
# GPU session: full -m gpu suite, then the profile round (bench line, launch list, ncu full capture), then C3/C4 bench lines.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
cp /root/repo/MEASURED_PEAKS.json gpurun_out/ 2>/dev/null
timeout 1800 python -m pytest tests/ -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 900 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1800 bash tools/profile_round.sh r01 ; echo prof=$?
for c in C3 C4; do
  timeout 1500 python bench.py --config $c --steps 10 --warmup 3 --json-out gpurun_out/bench_$c.json > gpurun_out/bench_$c.log 2>&1; echo $c=$?
done
