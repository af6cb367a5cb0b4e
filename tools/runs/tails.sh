mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "misaligned or 2pow24" > gpurun_out/tails.log 2>&1; tail -3 gpurun_out/tails.log
RESCCL_BENCH_ONE_DEVICE=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --nvls 1 --size-mb 64 > gpurun_out/bench_mp_nvls.json 2> gpurun_out/bench_mp_nvls.err; tail -c 1500 gpurun_out/bench_mp_nvls.json; tail -5 gpurun_out/bench_mp_nvls.err
