mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000
timeout 1800 python tools/sweep.py c2 nr > gpurun_out/sweep_c2_nr_head.jsonl 2>&1
wc -l gpurun_out/sweep_c2_nr_head.jsonl
