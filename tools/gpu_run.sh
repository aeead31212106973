#!/bin/bash
# The one runner for GPU sessions (gpurun -- 'tools/gpu_run.sh <cmd> ...'; several
# commands may be chained in one call).  Outputs go to gpurun_out/.
#   tests [pytest args]          pytest -m gpu (full GPU suite) -> pytest_gpu.log
#   bench C2 [bench args]        bench.py --config C2 [args] -> bench_C2.json / .log
#   ncu C2 L E                   ncu --set full of the bench's kernel on C2 at (L, E)
#   ncubuild [lib]               ncu --set full of one mid-build round_search and of phase1
#   launches                     ncu launch list of the default bench (the driver's recipe)
#   buildab LIB...               C2 build, Phase 1 / Phase 2 on the GPU clock, per library
#                                (variants from tools/variant.py), alternating twice
#   phases LIB C L E             per-phase cycle shares (GANNS_PROFILE library)
#   tail LIB                     per-round tail of the Phase-2 searches (GANNS_PROFILE library)
#   searchab C L LIB...          search A/B of libraries at one (config, l)
#   checks                       strong scaling under torchrun (NCCL, world 1), the
#                                reference arm, C5 on one GPU
set -u
mkdir -p gpurun_out
cmd=$1; shift
case "$cmd" in
  tests)
    timeout 3000 python -m pytest tests -m gpu -x -q -rA "$@" > gpurun_out/pytest_gpu.log 2>&1
    tail -5 gpurun_out/pytest_gpu.log ;;
  bench)
    cfg=$1; shift
    timeout 1500 python bench.py --config "$cfg" --json-out "gpurun_out/bench_${cfg}.json" "$@" \
      > "gpurun_out/bench_${cfg}.log" 2>&1
    echo "bench $cfg rc=$?"; tail -c 600 "gpurun_out/bench_${cfg}.log" ;;
  ncu)
    cfg=$1; l=$2; e=$3
    timeout 1500 ncu --set full --import-source on --clock-control none \
      -k "regex:^search(_group)?_kernel" -s 2 -c 1 \
      -o "gpurun_out/ncu_${cfg}_l${l}" -f python tools/prof_config.py --config "$cfg" --l "$l" --e "$e" \
      > "gpurun_out/ncu_${cfg}.log" 2>&1
    echo "ncu rc=$?"; tail -3 "gpurun_out/ncu_${cfg}.log" ;;
  ncubuild)
    lib=${1:-paper_conf_icde_yuwzqzl22_b200/libganns.so}
    GANNS_LIB_PATH=$lib timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_search \
      -s 350 -c 1 -o gpurun_out/ncu_round -f python tools/build_once.py > gpurun_out/ncu_round.log 2>&1
    GANNS_LIB_PATH=$lib timeout 900 ncu --set full --import-source on --clock-control none -k regex:phase1 \
      -s 1 -c 1 -o gpurun_out/ncu_phase1 -f python tools/build_once.py > gpurun_out/ncu_phase1.log 2>&1
    ls -la gpurun_out/ncu_round.ncu-rep gpurun_out/ncu_phase1.ncu-rep ;;
  launches)
    timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline \
      --proxy-worlds "" > gpurun_out/launches_bench.log 2>&1
    echo "launches rc=$?" ;;
  buildab)
    for rep in 1 2; do for lib in "$@"; do
      echo "== $lib"; GANNS_LIB_PATH=$lib timeout 600 python tools/build_phases.py 2 2>&1 | grep rep | tail -1
    done; done | tee -a gpurun_out/buildab.log ;;
  phases)
    GANNS_LIB_PATH=$1 timeout 900 python tools/phase_breakdown.py --config "$2" --l "$3" --e "$4" 2>&1 \
      | tail -1 | tee -a gpurun_out/phase_breakdown.log ;;
  tail)
    GANNS_LIB_PATH=$1 timeout 900 python tools/round_tail.py 2>&1 | tail -14 | tee -a gpurun_out/round_tail.log ;;
  searchab)
    cfg=$1; l=$2; shift 2
    for lib in "$@"; do
      GANNS_LIB_PATH=$lib timeout 900 python tools/search_ab.py --config "$cfg" --l "$l" 2>&1 | tail -1
    done | tee -a "gpurun_out/searchab_${cfg}.log" ;;
  checks)
    timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
      --master-port 29611 bench.py --gpus 1 --steps 10 --warmup 3 --scaling strong --no-cpu-baseline \
      > gpurun_out/strong_torchrun.log 2>&1; tail -c 400 gpurun_out/strong_torchrun.log
    timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/reference_arm.log 2>&1
    tail -c 600 gpurun_out/reference_arm.log
    timeout 1500 python bench.py --config C5 --shard-rows 1000000 --json-out gpurun_out/bench_C5.json \
      > gpurun_out/bench_C5.log 2>&1; tail -c 400 gpurun_out/bench_C5.log ;;
  *) echo "unknown command $cmd"; exit 2 ;;
esac
