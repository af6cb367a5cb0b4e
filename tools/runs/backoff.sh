mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
LAT_SIZES="[1024, 65536, 1048576, 16777216]" timeout 600 python tools/lat.py "instances=18 chunkbytes=8388608 direct=1" "instances=18 chunkbytes=8388608 direct=1 backoff=0" "instances=1 chunkbytes=8388608 direct=1 tma=0" "instances=1 chunkbytes=8388608 direct=1 tma=0 backoff=0" "instances=1 chunkbytes=8388608 direct=1 tma=0 nwarps=4" "instances=1 chunkbytes=8388608 direct=1 tma=0 nwarps=4 backoff=0" > gpurun_out/backoff_lat.jsonl 2>&1
cat gpurun_out/backoff_lat.jsonl
for v in 1 0; do RESCCL_BACKOFF=$v timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('backoff=$v', d['value'], d['config']['inplace_busbw_gbs'], d['sweep_busbw_gbs'])"; done
