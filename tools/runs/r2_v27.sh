mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
B="fifodepth=2 direct=1 linkmodel=port"
LAT_ALGO=hm LAT_GOPTS="g=8" LAT_SIZES="[4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "instances=18 chunkbytes=8388608 nwarps=8 $B" "instances=18 chunkbytes=1048576 nwarps=8 $B" "instances=18 chunkbytes=524288 nwarps=8 $B" "instances=18 chunkbytes=8388608 nwarps=16 tmatile=28672 $B" "instances=18 chunkbytes=8388608 nwarps=8 tmamin=65536 $B" "instances=18 chunkbytes=8388608 nwarps=8 lookahead=0 $B" > gpurun_out/r2v27_mesh.jsonl 2> gpurun_out/r2v27.err
cat gpurun_out/r2v27_mesh.jsonl | cut -c1-200; tail -2 gpurun_out/r2v27.err
