mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
A="instances=16 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1"
B="instances=18 nwarps=6 linkmodel=port chunkbytes=8388608 direct=1"
C="instances=18 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1"
D="instances=18 nwarps=4 linkmodel=port chunkbytes=8388608 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[16777216, 33554432, 67108864, 268435456]" timeout 1500 python tools/lat_graph.py "$A" "$B" "$C" "$D" "$A" "$B" "$C" "$D" > gpurun_out/lat_ab_classes.jsonl 2>&1
