# r02: per-SM HBM rate of the lane engine (ring AR, 256 MiB, 8 virtual ranks) at 8 / 16 / 24 CTAs
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
C="chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[268435456]" timeout 1200 python tools/lat_graph.py "instances=1 nwarps=8 $C" "instances=2 nwarps=8 $C" "instances=3 nwarps=8 $C" "instances=1 nwarps=16 $C" "instances=2 nwarps=16 $C" "instances=3 nwarps=16 $C" "instances=1 nwarps=8 bulkred=0 $C" > gpurun_out/r2v19_persm.jsonl 2> gpurun_out/r2v19.err
cat gpurun_out/r2v19_persm.jsonl
