#!/bin/bash
# Run on the GPU box (gpurun): bench line, ncu launch list of the bench command,
# one ncu --set full capture of the search kernel at the bench's l, summaries.
# Usage: bash tools/profile_round.sh <tag>
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
python bench.py --steps 10 --warmup 3 --json-out $OUT/bench_$TAG.json > $OUT/bench_$TAG.log 2>&1
L=$(python -c "import json;print(json.load(open('$OUT/bench_$TAG.json'))['config']['l'])")
E=$(python -c "import json;print(json.load(open('$OUT/bench_$TAG.json'))['config']['e'])")
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:^search_kernel --csv \
    --log-file $OUT/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline \
    > $OUT/launches_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:^search_kernel -s 2 -c 1 \
    -o $OUT/search_full_$TAG python tools/prof_search.py --l $L --e $E --l-build 128 > $OUT/ncu_$TAG.log 2>&1
python tools/ncu_summary.py $OUT/search_full_$TAG.ncu-rep > $OUT/ncu_summary_$TAG.json 2>&1
echo "bench l=$L e=$E"; tail -c 600 $OUT/bench_$TAG.json
