mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 > gpurun_out/gpu_tests10.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests10.log
export LAT_SIZES="[1024, 65536, 1048576, 16777216, 268435456]"
timeout 500 python tools/lat.py "instances=18 chunkbytes=8388608 direct=1" "instances=18 chunkbytes=8388608 direct=1 fuse=0" > gpurun_out/lat5.jsonl 2>&1
python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_fused.json 2>&1
