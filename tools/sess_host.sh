mkdir -p gpurun_out
python tools/alloc_probe.py > gpurun_out/alloc_probe.log 2>&1; cat gpurun_out/alloc_probe.log
timeout 600 python tools/build_phases.py 8 2>&1 | grep rep > gpurun_out/build_phases2.log; cat gpurun_out/build_phases2.log
