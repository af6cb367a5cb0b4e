mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000
timeout 1500 python tools/sweep.py c3w c4w > gpurun_out/sweep_c3w.jsonl 2>&1
cut -c1-250 gpurun_out/sweep_c3w.jsonl
