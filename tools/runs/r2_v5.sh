mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py -q -x -m gpu -k "direct or round_robin or fig16" > gpurun_out/r2v5_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v5_pytest.log
tail -3 gpurun_out/r2v5_pytest.log
B="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 67108864]" timeout 600 python tools/lat_graph.py "$B lookahead=0" "$B" "$B backoff=0" "instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" > gpurun_out/r2v5_lat.jsonl 2> gpurun_out/r2v5_lat.err
PHASE_OPTS="instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" timeout 300 python tools/phase_trace.py 1024 1048576 > gpurun_out/r2v5_phase_i1.jsonl 2> gpurun_out/r2v5_phase_i1.err
cat gpurun_out/r2v5_lat.jsonl
