mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py -q -x -m gpu -k "direct or round_robin or fig16 or graph" > gpurun_out/r2v6_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v6_pytest.log
tail -2 gpurun_out/r2v6_pytest.log
B="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 67108864]" timeout 600 python tools/lat_graph.py "$B lookahead=0" "$B" "$B pollacq=1" "$B backoff=0" "$B lookahead=0 relaybypass=0" > gpurun_out/r2v6_lat.jsonl 2> gpurun_out/r2v6_lat.err
C="nwarps=8 fifodepth=2 direct=1"
LAT_SIZES="[16777216, 67108864]" timeout 900 python tools/lat_graph.py "instances=14 chunkbytes=1048576 $C" "instances=14 chunkbytes=524288 $C" "instances=7 chunkbytes=1048576 $C" "instances=7 chunkbytes=524288 $C" "instances=7 chunkbytes=2097152 $C" "instances=14 chunkbytes=4194304 $C" "instances=14 chunkbytes=2097152 $C" "instances=18 chunkbytes=2097152 $C" > gpurun_out/r2v6_pipe.jsonl 2> gpurun_out/r2v6_pipe.err
PHASE_OPTS="instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" timeout 300 python tools/phase_trace.py 1024 > gpurun_out/r2v6_phase_i1.jsonl 2> gpurun_out/r2v6_phase_i1.err
cat gpurun_out/r2v6_lat.jsonl gpurun_out/r2v6_pipe.jsonl
