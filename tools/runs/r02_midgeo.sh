# mid-size (4-64 MiB) geometry search for the size-tuned AllReduce
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=()
for i in 14 16 18; do for cb in 2097152 8388608; do O+=("instances=$i nwarps=8 linkmodel=port chunkbytes=$cb direct=1"); O+=("instances=$i nwarps=12 tmatile=28672 linkmodel=port chunkbytes=$cb direct=1"); done; done
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[4194304, 16777216, 67108864]" timeout 1200 python tools/lat_graph.py "${O[@]}" > gpurun_out/lat_midgeo.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="[4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "instances=4 nwarps=8 chunkbytes=1048576 direct=1" "instances=4 nwarps=12 tmatile=28672 chunkbytes=1048576 direct=1" "instances=18 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1" >> gpurun_out/lat_midgeo.jsonl 2>&1
LAT_SIZES="[4194304, 16777216, 67108864]" timeout 600 python tools/lat_graph.py "instances=18 nwarps=8 chunkbytes=33554432 direct=1" "instances=18 nwarps=8 chunkbytes=2097152 direct=1" >> gpurun_out/lat_midgeo.jsonl 2>&1
wc -l gpurun_out/lat_midgeo.jsonl
