#!/bin/bash
# Round-end measurement set: GPU suite, smoke, bench lines C2-C5, profile of the C2 search kernel
mkdir -p gpurun_out/final
O=gpurun_out/final
timeout 2000 python -m pytest tests/ -q -m gpu > $O/pytest_gpu.log 2>&1; echo pytest=$?; tail -1 $O/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py --json-out $O/bench_C2.json > $O/bench_C2.log 2>&1; echo C2=$?
for c in C3 C4; do timeout 1200 python bench.py --config $c --json-out $O/bench_$c.json > $O/bench_$c.log 2>&1; echo $c=$?; done
L=$(python -c "import json;print(json.load(open('$O/bench_C2.json'))['config']['l'])")
E=$(python -c "import json;print(json.load(open('$O/bench_C2.json'))['config']['e'])")
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:^search_kernel --csv --log-file $O/launches_C2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $O/launches.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:^search_kernel -s 2 -c 1 -o $O/search_full python tools/prof_search.py --l $L --e $E --l-build 128 > $O/ncu.log 2>&1
python tools/ncu_summary.py $O/search_full.ncu-rep > $O/ncu_summary.json 2>&1
timeout 3000 python bench.py --config C5 --steps 5 --warmup 3 --json-out $O/bench_C5.json > $O/bench_C5.log 2>&1; echo C5=$?
