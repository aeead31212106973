mkdir -p gpurun_out
python tools/build_once.py C2 6 > gpurun_out/build_times.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/build_launches.csv python tools/build_once.py > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:round_search -s 300 -c 1 -o gpurun_out/ncu_round -f python tools/build_once.py > gpurun_out/ncu_round.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:phase1 -s 1 -c 1 -o gpurun_out/ncu_phase1 -f python tools/build_once.py > gpurun_out/ncu_phase1.log 2>&1
cat gpurun_out/build_times.log; tail -2 gpurun_out/ncu_round.log gpurun_out/ncu_phase1.log
