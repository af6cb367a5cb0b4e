mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
B="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 67108864]" timeout 600 python tools/lat_graph.py "$B lookahead=0" "$B" "instances=18 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" > gpurun_out/r2v7_lat.jsonl 2> gpurun_out/r2v7_lat.err
timeout 1500 python tools/sweep.py geo > gpurun_out/r2v7_geo.jsonl 2> gpurun_out/r2v7_geo.err
cat gpurun_out/r2v7_lat.jsonl; tail -3 gpurun_out/r2v7_geo.err
