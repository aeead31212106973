mkdir -p gpurun_out
for lib in paper_conf_icde_yuwzqzl22_b200/libganns.so ab/libganns_p0.so; do
  echo "== $lib"; GANNS_LIB_PATH=$lib timeout 600 python tools/build_phases.py 8 2>&1 | grep rep
done > gpurun_out/build_phases.log
cat gpurun_out/build_phases.log
tools/gpu_run.sh bench C3
