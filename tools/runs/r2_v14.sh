mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
B="nwarps=8 fifodepth=2 direct=1"
SZ="[262144, 1048576, 4194304, 16777216, 67108864, 268435456]"
LAT_ALGO=hm LAT_GOPTS="g=8" LAT_SIZES="$SZ" timeout 1500 python tools/lat_graph.py "instances=2 chunkbytes=33554432 tmamin=262144 $B" "instances=18 chunkbytes=2097152 linkmodel=port $B" "instances=18 chunkbytes=33554432 linkmodel=port $B" "instances=14 chunkbytes=8388608 linkmodel=port $B" "instances=18 chunkbytes=8388608 linkmodel=port $B" > gpurun_out/r2v14_mesh.jsonl 2> gpurun_out/r2v14.err
tail -3 gpurun_out/r2v14.err
