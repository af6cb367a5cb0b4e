mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
B="fifodepth=2 direct=1"
LAT_ALGO=hm LAT_GOPTS="g=8" LAT_SIZES="[4194304, 16777216, 67108864, 268435456]" timeout 900 python tools/lat_graph.py "instances=18 chunkbytes=8388608 nwarps=12 tmatile=28672 linkmodel=port $B" "instances=12 chunkbytes=8388608 nwarps=12 tmatile=28672 linkmodel=port $B" "instances=14 chunkbytes=8388608 nwarps=12 tmatile=28672 linkmodel=port $B" > gpurun_out/r2v33.jsonl 2> gpurun_out/r2v33.err
LAT_ALGO=dbt LAT_SIZES="[268435456]" timeout 900 python tools/lat_graph.py "instances=18 chunkbytes=8388608 nwarps=12 tmatile=28672 linkmodel=port $B" >> gpurun_out/r2v33.jsonl 2>> gpurun_out/r2v33.err
LAT_ALGO=hm LAT_GOPTS="g=4" LAT_SIZES="[268435456]" timeout 900 python tools/lat_graph.py "instances=4 chunkbytes=1048576 nwarps=12 tmatile=28672 $B" >> gpurun_out/r2v33.jsonl 2>> gpurun_out/r2v33.err
cat gpurun_out/r2v33.jsonl | cut -c1-220; tail -2 gpurun_out/r2v33.err
