# r02: the torchrun (N>1) bench path end to end with 2 processes on one GPU (CUDA IPC):
# TB-utilisation summary, NCCL comparison (expected to fail: one device), tuned sweep
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py tests/test_gpu_multiprocess.py -q -x -m gpu -k "direct or registered or pushreduce" > gpurun_out/r2v18_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v18_pytest.log
tail -2 gpurun_out/r2v18_pytest.log
export RESCCL_BENCH_ONE_DEVICE=1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 2 --steps 5 --warmup 3 --size-mb 64 --e2e-steps 1 > gpurun_out/r2v18_bench_mp2.json 2> gpurun_out/r2v18_bench_mp2.err
tail -c 3000 gpurun_out/r2v18_bench_mp2.json; grep -v "^\s*$" gpurun_out/r2v18_bench_mp2.err | grep -i "error" | tail -5
