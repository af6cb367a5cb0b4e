# C2/C3/C4/f2 sweeps under the 24 KiB-tile geometry (direct transport)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 1200 python tools/sweep.py c2 > gpurun_out/sweep_c2_v8.jsonl 2>&1
timeout 900 python tools/sweep.py c3 c4 f2 > gpurun_out/sweep_c3c4f2_v8.jsonl 2>&1
wc -l gpurun_out/sweep_*_v8.jsonl
