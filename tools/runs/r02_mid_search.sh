mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 2400 python tools/mid_search.py > gpurun_out/mid_search.jsonl 2>&1
grep -c graph_us gpurun_out/mid_search.jsonl
