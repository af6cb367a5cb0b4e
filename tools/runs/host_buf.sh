# host-buffer collectives: GPU tests + bench e2e under the library-staged path
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python -m pytest tests/test_gpu_host_buffers.py -x -q > gpurun_out/pytest_host.log 2>&1
echo "pytest=$?" >> gpurun_out/pytest_host.log
tail -15 gpurun_out/pytest_host.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_host.json 2> gpurun_out/bench_host.err
cat gpurun_out/bench_host.json; tail -5 gpurun_out/bench_host.err
for p in 8388608 67108864 268435456; do
  RESCCL_HOST_PIECE=$p timeout 300 python bench.py --no-cpu-baseline --steps 3 --warmup 3 --e2e-steps 5 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print($p, d['e2e'])"
done
