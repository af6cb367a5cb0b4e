# r02: C5 analogue (25 MiB bf16 AllReduce buckets concurrent with an 8192^3 bf16 GEMM loop)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
OVERLAP_OPTS="chunkbytes=33554432 nwarps=8 direct=1" timeout 900 python tools/overlap.py > gpurun_out/r2v26_overlap_ring.jsonl 2> gpurun_out/r2v26.err
OVERLAP_ALGO=hm OVERLAP_GOPTS="g=8" OVERLAP_OPTS="chunkbytes=8388608 nwarps=8 linkmodel=port direct=1" timeout 900 python tools/overlap.py > gpurun_out/r2v26_overlap_mesh.jsonl 2>> gpurun_out/r2v26.err
cat gpurun_out/r2v26_overlap_ring.jsonl gpurun_out/r2v26_overlap_mesh.jsonl; tail -3 gpurun_out/r2v26.err
