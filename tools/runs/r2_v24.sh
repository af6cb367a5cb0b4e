mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
PHASE_ALGO=hm PHASE_GOPTS="g=8" PHASE_OPTS="instances=1 nwarps=8 chunkbytes=2097152 fifodepth=2 direct=1" timeout 300 python tools/phase_trace.py 1024 65536 > gpurun_out/r2v24_phase_mesh.jsonl 2> gpurun_out/r2v24.err
PHASE_ALGO=hm PHASE_GOPTS="g=8" PHASE_OPTS="instances=1 nwarps=8 chunkbytes=2097152 fifodepth=2 direct=1 linkmodel=port" timeout 300 python tools/phase_trace.py 1024 > gpurun_out/r2v24_phase_mesh_port.jsonl 2>> gpurun_out/r2v24.err
tail -3 gpurun_out/r2v24.err
