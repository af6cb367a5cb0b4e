# r02: per-SM rate vs warps / tile / stages at 8 CTAs (ring AR 256 MiB, out of place)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
C="instances=1 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[268435456]" timeout 1200 python tools/lat_graph.py "$C nwarps=16 tmatile=28672" "$C nwarps=32 tmatile=28672" "$C nwarps=16 tmatile=57344 tmastages=1" "$C nwarps=32 tmatile=57344 tmastages=1" "$C nwarps=16 tmatile=18944 tmastages=3" "$C nwarps=32 tmatile=18944 tmastages=3" "$C nwarps=24 tmatile=28672" > gpurun_out/r2v29_persm.jsonl 2> gpurun_out/r2v29.err
C3="instances=3 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[268435456]" timeout 600 python tools/lat_graph.py "$C3 nwarps=16 tmatile=28672" "$C3 nwarps=32 tmatile=28672" >> gpurun_out/r2v29_persm.jsonl 2>> gpurun_out/r2v29.err
tail -3 gpurun_out/r2v29.err
