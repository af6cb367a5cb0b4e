# torchrun, 2 processes on the one GPU: the multi-process bench path incl. host-buffer e2e
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000 RESCCL_BENCH_ONE_DEVICE=1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29522 bench.py --gpus 2 --steps 3 --warmup 3 --size-mb 32 > gpurun_out/mp_e2e.json 2> gpurun_out/mp_e2e.err
echo "rc=$?"; cat gpurun_out/mp_e2e.json; tail -3 gpurun_out/mp_e2e.err
