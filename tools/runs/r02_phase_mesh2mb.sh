mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
PHASE_ALGO=hm PHASE_GOPTS=g=8 PHASE_RAW=gpurun_out/phase_raw_mesh2mb.jsonl PHASE_OPTS="instances=18 nwarps=8 linkmodel=port chunkbytes=1048576 direct=1" timeout 300 python tools/phase_trace.py 16777216 > gpurun_out/phase_mesh2mb.jsonl 2>&1
