# per-primitive setup gap: phase timelines and graph latency with / without descriptor warm-up
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
for dw in 0 1; do
  PHASE_RAW=gpurun_out/phase_raw_dw$dw.jsonl PHASE_OPTS="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1 descwarm=$dw" timeout 300 python tools/phase_trace.py 1024 16777216 >> gpurun_out/phase_dw.jsonl 2>&1
done
LAT_SIZES="[1024, 1048576, 16777216, 67108864, 268435456]" timeout 900 python tools/lat_graph.py "instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" "instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1 descwarm=1" > gpurun_out/lat_dw.jsonl 2>&1
cat gpurun_out/lat_dw.jsonl
