mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
LAT_SIZES="[1024, 65536, 1048576, 16777216]" timeout 600 python tools/lat.py "instances=18 chunkbytes=8388608 direct=1" "instances=18 chunkbytes=8388608 direct=1 pollacq=1" "instances=1 chunkbytes=8388608 direct=1" "instances=1 chunkbytes=8388608 direct=1 pollacq=1" "instances=18 chunkbytes=4194304 direct=0" "instances=18 chunkbytes=4194304 direct=0 pollacq=1" > gpurun_out/pollacq_lat.jsonl 2>&1
cat gpurun_out/pollacq_lat.jsonl
for v in 0 1; do RESCCL_POLL_ACQ=$v timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --sweep 1,16,64 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('pollacq=$v', d['value'], d['config']['inplace_busbw_gbs'], d['sweep_busbw_gbs'])"; done
