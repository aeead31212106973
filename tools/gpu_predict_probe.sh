timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/t5_all.log 2>&1; echo tests=$?
bash tools/ab_bench.sh 112,128 > gpurun_out/ab_predict.log 2>&1
