mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=()
for i in 14 16 18; do for w in 4 6; do O+=("instances=$i nwarps=$w linkmodel=port chunkbytes=8388608 direct=1"); done; done
O+=("instances=16 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1")
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[33554432, 67108864, 268435456]" timeout 1200 python tools/lat_graph.py "${O[@]}" > gpurun_out/lat_warps_big.jsonl 2>&1
LAT_SIZES="[16777216, 268435456]" timeout 900 python tools/lat_graph.py "instances=12 nwarps=12 tmatile=28672 chunkbytes=33554432 direct=1" "instances=12 nwarps=8 tmatile=28672 chunkbytes=33554432 direct=1" "instances=12 nwarps=6 tmatile=28672 chunkbytes=33554432 direct=1" >> gpurun_out/lat_warps_big.jsonl 2>&1
