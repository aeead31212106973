mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_search -s 300 -c 1 -o gpurun_out/ncu_round_r02b -f python tools/build_once.py > gpurun_out/ncu_round_r02b.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:phase1 -s 1 -c 1 -o gpurun_out/ncu_phase1_r02b -f python tools/build_once.py > gpurun_out/ncu_phase1_r02b.log 2>&1
ls -la gpurun_out/*r02b*
