mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
PHASE_ALGO=hm PHASE_GOPTS=g=8 PHASE_RAW=gpurun_out/phase_raw_meshpair.jsonl PHASE_OPTS="instances=1 nwarps=8 chunkbytes=33554432 direct=1" timeout 300 python tools/phase_trace.py 1024 > gpurun_out/phase_meshpair.jsonl 2>&1
