mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
B="instances=12 nwarps=12 tmatile=28672 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[16777216, 67108864, 268435456]" timeout 1200 python tools/lat_graph.py "$B" "$B cpoll=1" "$B" "$B cpoll=1" > gpurun_out/lat_cpoll.jsonl 2>&1
M="instances=18 linkmodel=port chunkbytes=8388608 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[16777216, 33554432, 268435456]" timeout 1200 python tools/lat_graph.py "$M nwarps=4" "$M nwarps=8 cpoll=1" "$M nwarps=8" "instances=16 linkmodel=port chunkbytes=8388608 direct=1 nwarps=8 cpoll=1" "instances=16 linkmodel=port chunkbytes=8388608 direct=1 nwarps=8" >> gpurun_out/lat_cpoll.jsonl 2>&1
