# two CTAs per SM for the mid-size mesh: smaller TMA pools, more instances
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=("instances=18 nwarps=4 linkmodel=port chunkbytes=8388608 direct=1")
for i in 27 36; do for t in 12288 14336; do O+=("instances=$i nwarps=4 tmatile=$t linkmodel=port chunkbytes=8388608 direct=1"); done; done
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[4194304, 8388608, 16777216, 33554432]" timeout 1500 python tools/lat_graph.py "${O[@]}" > gpurun_out/lat_two_per_sm.jsonl 2>&1
