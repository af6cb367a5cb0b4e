mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000
timeout 900 python tools/overlap.py > gpurun_out/overlap_head2.jsonl 2>&1
cat gpurun_out/overlap_head2.jsonl | cut -c1-300
