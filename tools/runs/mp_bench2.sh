mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000 RESCCL_BENCH_ONE_DEVICE=1
nvidia-cuda-mps-control -d && echo mps-started
P=29600
for np in 2 4; do
 for d in 1 0; do
  P=$((P+1))
  echo "np=$np direct=$d" >> gpurun_out/mp_bench2.txt
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $np --master-addr 127.0.0.1 --master-port $P bench.py --gpus $np --steps 5 --warmup 3 --size-mb 64 --direct $d --e2e-steps 0 --no-cpu-baseline 2>> gpurun_out/mp_bench2.err | tail -1 >> gpurun_out/mp_bench2.txt
 done
done
echo quit | nvidia-cuda-mps-control
