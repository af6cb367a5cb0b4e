# r02: per-SM HBM rate variants at 8 CTAs (ring AR 256 MiB): protocol options, tile sizes
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
C="instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[268435456]" timeout 1200 python tools/lat_graph.py "$C" "$C lookahead=0" "$C lookahead=0 relaybypass=0" "$C tmatile=28672" "$C tmatile=16384 tmastages=3" "$C tmatile=28672 lookahead=0" "$C nwarps=16 tmatile=28672" > gpurun_out/r2v20_persm.jsonl 2> gpurun_out/r2v20.err
C14="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[16777216, 268435456]" timeout 600 python tools/lat_graph.py "$C14" "$C14 tmatile=28672" >> gpurun_out/r2v20_persm.jsonl 2>> gpurun_out/r2v20.err
cat gpurun_out/r2v20_persm.jsonl; tail -3 gpurun_out/r2v20.err
