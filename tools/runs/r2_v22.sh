mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
timeout 1500 python tools/sweep.py c3 > gpurun_out/r2v22_c3.jsonl 2> gpurun_out/r2v22_c3.err
tail -3 gpurun_out/r2v22_c3.err
