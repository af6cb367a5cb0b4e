mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v12.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_v12.log
python bench.py > gpurun_out/bench_v12.json 2> gpurun_out/bench_v12.err
timeout 1200 python tools/sweep.py c2 > gpurun_out/sweep_c2_v12.jsonl 2>&1
tail -3 gpurun_out/pytest_gpu_v12.log; head -c 600 gpurun_out/bench_v12.json
