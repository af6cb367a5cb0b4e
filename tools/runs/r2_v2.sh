# r02: phase breakdown of ring AR (8 virtual ranks) at 1 KiB / 1 MiB / 16 MiB; torch backend test
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python tools/phase_trace.py 1024 1048576 16777216 > gpurun_out/r2v2_phase_bench.jsonl 2> gpurun_out/r2v2_phase_bench.err
PHASE_OPTS="instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" timeout 600 python tools/phase_trace.py 1024 1048576 > gpurun_out/r2v2_phase_i1.jsonl 2> gpurun_out/r2v2_phase_i1.err
PHASE_OPTS="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=0" timeout 600 python tools/phase_trace.py 1024 16777216 > gpurun_out/r2v2_phase_staged.jsonl 2> gpurun_out/r2v2_phase_staged.err
timeout 600 python -m pytest tests/test_gpu_process_group.py -q -x > gpurun_out/r2v2_pg.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v2_pg.log
tail -3 gpurun_out/r2v2_pg.log; tail -3 gpurun_out/r2v2_phase_bench.err
