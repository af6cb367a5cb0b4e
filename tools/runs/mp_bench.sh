mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000 RESCCL_BENCH_ONE_DEVICE=1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 3 --warmup 3 --size-mb 32 > gpurun_out/mp_bench.json 2> gpurun_out/mp_bench.err
echo rc=$? >> gpurun_out/mp_bench.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/mp_ref.json 2> gpurun_out/mp_ref.err
echo rc=$? >> gpurun_out/mp_ref.err
nvidia-cuda-mps-control -d && echo mps-started
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29514 bench.py --gpus 2 --steps 5 --warmup 3 --size-mb 64 > gpurun_out/mp_bench_mps.json 2> gpurun_out/mp_bench_mps.err
echo rc=$? >> gpurun_out/mp_bench_mps.err
echo quit | nvidia-cuda-mps-control
