# HEAD: the torchrun (N>1) bench path end to end with 2 processes on one GPU (CUDA IPC)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
export RESCCL_BENCH_ONE_DEVICE=1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 2 --steps 5 --warmup 3 --size-mb 64 --e2e-steps 1 > gpurun_out/mp2_head.json 2> gpurun_out/mp2_head.err
echo "rc=$?"; tail -c 2500 gpurun_out/mp2_head.json; grep -i "error\|Traceback" gpurun_out/mp2_head.err | tail -5
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29542 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/mp2_ref.json 2> gpurun_out/mp2_ref.err; echo "ref rc=$?"; tail -c 600 gpurun_out/mp2_ref.json
