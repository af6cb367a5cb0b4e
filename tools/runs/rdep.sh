mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
LAT_SIZES="[1024, 65536, 1048576, 4194304, 16777216, 67108864]" timeout 600 python tools/lat.py "instances=18 chunkbytes=8388608 direct=1" "instances=18 chunkbytes=8388608 direct=1 rdep=1" "instances=1 chunkbytes=8388608 direct=1" "instances=1 chunkbytes=8388608 direct=1 rdep=1" > gpurun_out/rdep_lat.jsonl 2>&1
cat gpurun_out/rdep_lat.jsonl | grep -v Warn
for v in 0 1; do RESCCL_RDEP=$v timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rdep=$v', d['value'], d['config']['inplace_busbw_gbs'], d['sweep_busbw_gbs'], d['async_error'])"; done
RESCCL_RDEP=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_multiprocess.py -x -q > gpurun_out/pytest_rdep.log 2>&1; echo "pytest_rdep=$?" >> gpurun_out/pytest_rdep.log
tail -3 gpurun_out/pytest_rdep.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v16.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_v16.log
tail -3 gpurun_out/pytest_gpu_v16.log
