#!/bin/bash
# One documented runner for GPU sessions (replaces the round-1 one-shot scripts).
#   tools/gpu_run.sh tests            pytest -m gpu (full GPU suite)
#   tools/gpu_run.sh bench C2 [args]  bench.py --config C2 [args] -> gpurun_out/bench_C2.json
#   tools/gpu_run.sh ncu C2 L E       ncu --set full of the bench's kernel on config C2 at (L, E)
#   tools/gpu_run.sh launches         ncu launch list of the default bench (driver's recipe)
set -u
mkdir -p gpurun_out
case "$1" in
  tests)
    shift
    timeout 3000 python -m pytest tests -m gpu -x -q -rA "$@" > gpurun_out/pytest_gpu.log 2>&1
    tail -5 gpurun_out/pytest_gpu.log ;;
  bench)
    cfg=$2; shift 2
    timeout 1500 python bench.py --config "$cfg" --json-out "gpurun_out/bench_${cfg}.json" "$@" \
      > "gpurun_out/bench_${cfg}.log" 2>&1
    echo "bench $cfg rc=$?"; tail -c 600 "gpurun_out/bench_${cfg}.log" ;;
  ncu)
    cfg=$2; l=$3; e=$4
    timeout 1500 ncu --set full --import-source on --clock-control none \
      -k "regex:^search(_group)?_kernel" -s 2 -c 1 \
      -o "gpurun_out/ncu_${cfg}_l${l}" -f python tools/prof_config.py --config "$cfg" --l "$l" --e "$e" \
      > "gpurun_out/ncu_${cfg}.log" 2>&1
    echo "ncu rc=$?"; tail -3 "gpurun_out/ncu_${cfg}.log" ;;
  launches)
    timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline \
      --proxy-worlds "" > gpurun_out/launches_bench.log 2>&1
    echo "launches rc=$?" ;;
esac
