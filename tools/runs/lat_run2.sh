export RESCCL_TIMEOUT_MS=10000
export LAT_SIZES="[16777216, 33554432, 67108864, 134217728, 268435456]"
timeout 500 python tools/lat.py "instances=18 chunkbytes=8388608 direct=1 tmamin=0" "instances=18 chunkbytes=8388608 direct=1 tma=0" "instances=18 chunkbytes=4194304 direct=0 tmamin=0" "instances=18 chunkbytes=4194304 direct=0 tma=0" > gpurun_out/lat4.jsonl 2>&1
