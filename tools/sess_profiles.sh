# round-2 ncu evidence: launch list of the default bench command (driver recipe), one
# --set full capture of the bench kernel per config at its operating point, one mid-build
# round_search and phase1 capture.
mkdir -p gpurun_out
tools/gpu_run.sh launches
tools/gpu_run.sh ncu C2 128 109
tools/gpu_run.sh ncu C3 288 288
tools/gpu_run.sh ncu C4 288 288
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_search -s 300 -c 1 -o gpurun_out/ncu_round_r02 -f python tools/build_once.py > gpurun_out/ncu_round_r02.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:phase1 -s 1 -c 1 -o gpurun_out/ncu_phase1_r02 -f python tools/build_once.py > gpurun_out/ncu_phase1_r02.log 2>&1
ls -la gpurun_out/*.ncu-rep
