mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=()
for w in 4 6 8; do O+=("instances=18 nwarps=$w linkmodel=port chunkbytes=8388608 direct=1"); done
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[8388608, 16777216, 33554432, 67108864]" timeout 900 python tools/lat_graph.py "${O[@]}" > gpurun_out/lat_warps_mid.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="[2097152, 4194304, 8388608]" timeout 900 python tools/lat_graph.py "instances=4 nwarps=6 chunkbytes=524288 direct=1" "instances=4 nwarps=8 chunkbytes=524288 direct=1" "instances=4 nwarps=4 chunkbytes=524288 direct=1" >> gpurun_out/lat_warps_mid.jsonl 2>&1
