# r02: phase breakdown again (raw times, graph replay), torch backend + NCCL shim tests
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python -m pytest tests/test_gpu_process_group.py tests/test_nccl_shim.py -q > gpurun_out/r2v3_f4.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v3_f4.log
PHASE_OPTS="instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" timeout 600 python tools/phase_trace.py 1024 1048576 > gpurun_out/r2v3_phase_i1.jsonl 2> gpurun_out/r2v3_phase_i1.err
timeout 600 python tools/phase_trace.py 1024 1048576 16777216 > gpurun_out/r2v3_phase_bench.jsonl 2> gpurun_out/r2v3_phase_bench.err
tail -3 gpurun_out/r2v3_f4.log; tail -3 gpurun_out/r2v3_phase_i1.err
