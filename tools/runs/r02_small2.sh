mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
S="[1024, 16384, 65536, 131072, 262144]"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="$S" timeout 600 python tools/lat_graph.py "instances=1 nwarps=2 chunkbytes=33554432 direct=1" "instances=1 nwarps=4 chunkbytes=33554432 direct=1" "instances=2 nwarps=4 chunkbytes=33554432 direct=1" > gpurun_out/lat_small2.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="$S" timeout 600 python tools/lat_graph.py "instances=4 nwarps=4 chunkbytes=524288 direct=1" "instances=4 nwarps=8 chunkbytes=524288 direct=1" "instances=2 nwarps=4 chunkbytes=524288 direct=1" >> gpurun_out/lat_small2.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="[1048576, 4194304]" timeout 600 python tools/lat_graph.py "instances=4 nwarps=4 chunkbytes=524288 direct=1" "instances=4 nwarps=8 chunkbytes=524288 direct=1" >> gpurun_out/lat_small2.jsonl 2>&1
