timeout 1200 python -m pytest tests/test_gpu_sanitizer.py tests/test_gpu_parity.py -x -q > gpurun_out/t6_san.log 2>&1; echo san=$?
for c in C2 C3 C4; do
  timeout 1500 python bench.py --config $c --steps 10 --warmup 3 --json-out gpurun_out/bench_$c.json > gpurun_out/bench_$c.log 2>&1; echo $c=$?
done
