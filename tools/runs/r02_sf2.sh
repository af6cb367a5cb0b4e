mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
M="instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1"
R="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
PHASE_ALGO=hm PHASE_GOPTS=g=8 PHASE_RAW=gpurun_out/phase_raw_sf2_mesh.jsonl PHASE_OPTS="$M splitfence=2" timeout 300 python tools/phase_trace.py 16777216 > /dev/null 2>&1
PHASE_RAW=gpurun_out/phase_raw_sf2_ring.jsonl PHASE_OPTS="$R splitfence=2" timeout 300 python tools/phase_trace.py 16777216 > /dev/null 2>&1
LAT_SIZES="[1024, 1048576, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "$R" "$R splitfence=2" > gpurun_out/lat_sf2.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1024, 4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "$M" "$M splitfence=2" "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=1 nwarps=8 chunkbytes=33554432 direct=1 splitfence=2" >> gpurun_out/lat_sf2.jsonl 2>&1
cut -c1-200 gpurun_out/lat_sf2.jsonl
