mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
C="instances=1 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[268435456]" timeout 1200 python tools/lat_graph.py "$C nwarps=16 tmatile=28672 cpoll=1" "$C nwarps=24 tmatile=28672 cpoll=1" "$C nwarps=32 tmatile=28672 cpoll=1" "$C nwarps=16 tmatile=57344 tmastages=1 cpoll=1" "$C nwarps=12 tmatile=28672" "$C nwarps=20 tmatile=28672" > gpurun_out/r2v30_persm.jsonl 2> gpurun_out/r2v30.err
tail -3 gpurun_out/r2v30.err
