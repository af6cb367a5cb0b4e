# phase timelines with 1 vs several micro-batches per hop (ring, 14 instances, 16 MiB)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
for cb in 33554432 1048576; do
  PHASE_RAW=gpurun_out/phase_raw_cb$cb.jsonl PHASE_OPTS="instances=14 nwarps=8 chunkbytes=$cb fifodepth=2 direct=1" timeout 300 python tools/phase_trace.py 16777216 >> gpurun_out/phase_mb.jsonl 2>&1
done
ls -la gpurun_out
