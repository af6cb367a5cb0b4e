# r02: DBT-8 under the port link model (one duplex CTA per rank x instances) vs pair
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
B="nwarps=8 fifodepth=2 direct=1"
LAT_ALGO=dbt LAT_SIZES="[16777216, 67108864, 268435456]" timeout 1500 python tools/lat_graph.py "instances=6 chunkbytes=8388608 $B" "instances=18 chunkbytes=8388608 linkmodel=port $B" "instances=18 chunkbytes=2097152 linkmodel=port $B" "instances=18 chunkbytes=33554432 linkmodel=port $B" "instances=12 chunkbytes=8388608 linkmodel=port $B" "instances=6 chunkbytes=4194304 nwarps=16 tmatile=28672 fifodepth=2 direct=1" > gpurun_out/r2v21_dbt.jsonl 2> gpurun_out/r2v21.err
cat gpurun_out/r2v21_dbt.jsonl | cut -c1-200; tail -3 gpurun_out/r2v21.err
