# small-message schedule search (1 KiB - 256 KiB): mesh, 2x4 / 4x2 hierarchical, DBT, ring
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
S="[1024, 16384, 65536, 262144]"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="$S" timeout 600 python tools/lat_graph.py "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=2 nwarps=8 chunkbytes=2097152 direct=1" "instances=1 nwarps=4 chunkbytes=33554432 direct=1" > gpurun_out/lat_small.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="$S" timeout 600 python tools/lat_graph.py "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=2 nwarps=8 chunkbytes=524288 direct=1" "instances=4 nwarps=8 chunkbytes=524288 direct=1" >> gpurun_out/lat_small.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=2 LAT_SIZES="$S" timeout 600 python tools/lat_graph.py "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=2 nwarps=8 chunkbytes=524288 direct=1" >> gpurun_out/lat_small.jsonl 2>&1
LAT_ALGO=dbt LAT_GOPTS="" LAT_SIZES="$S" timeout 600 python tools/lat_graph.py "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=2 nwarps=8 chunkbytes=33554432 direct=1" >> gpurun_out/lat_small.jsonl 2>&1
