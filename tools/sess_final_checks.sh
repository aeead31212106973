mkdir -p gpurun_out
tools/gpu_run.sh ncu C2 128 109
tools/gpu_run.sh ncu C3 288 288
tools/gpu_run.sh ncu C4 288 288
# code paths: strong scaling under torchrun (NCCL, world 1), the reference arm
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 1 --steps 10 --warmup 3 --scaling strong --no-cpu-baseline > gpurun_out/strong_torchrun.log 2>&1; tail -c 400 gpurun_out/strong_torchrun.log
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/reference_arm.log 2>&1; tail -c 600 gpurun_out/reference_arm.log
tools/gpu_run.sh bench C5 --shard-rows 1000000
