mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
PHASE_ALGO=hm PHASE_GOPTS=g=8 PHASE_RAW=gpurun_out/phase_raw_fine_mesh.jsonl PHASE_OPTS="instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1" timeout 300 python tools/phase_trace.py 16777216 > gpurun_out/phase_fine_mesh.jsonl 2>&1
PHASE_RAW=gpurun_out/phase_raw_fine_ring.jsonl PHASE_OPTS="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" timeout 300 python tools/phase_trace.py 16777216 > gpurun_out/phase_fine_ring.jsonl 2>&1
ls -la gpurun_out | tail -4
