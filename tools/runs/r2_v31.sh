mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
C="instances=1 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[268435456]" timeout 1200 python tools/lat_graph.py "$C nwarps=12 tmatile=24576" "$C nwarps=12 tmatile=57344 tmastages=1" "$C nwarps=14 tmatile=28672" "$C nwarps=10 tmatile=28672" "instances=3 chunkbytes=33554432 fifodepth=2 direct=1 nwarps=12 tmatile=28672" > gpurun_out/r2v31_persm.jsonl 2> gpurun_out/r2v31.err
B="chunkbytes=33554432 fifodepth=2 direct=1 nwarps=12 tmatile=28672"
LAT_SIZES="[16777216, 67108864, 268435456]" timeout 1200 python tools/lat_graph.py "instances=14 $B" "instances=10 $B" "instances=8 $B" "instances=12 $B" "instances=18 $B" "instances=14 chunkbytes=33554432 fifodepth=2 direct=1 nwarps=8" > gpurun_out/r2v31_cta.jsonl 2>> gpurun_out/r2v31.err
tail -3 gpurun_out/r2v31.err
