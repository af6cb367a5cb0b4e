# r02: relay bypass (R29) + writable lookahead (R30): parity first, then device-clock latency A/B
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py tests/test_gpu_process_group.py tests/test_nccl_shim.py -q -x -m gpu > gpurun_out/r2v4_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v4_pytest.log
timeout 900 python -m pytest tests/test_gpu_multiprocess.py -q -x -k "registered or graph" > gpurun_out/r2v4_pytest_mp.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v4_pytest_mp.log
B="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
timeout 900 python tools/lat_graph.py "$B relaybypass=0 lookahead=0" "$B lookahead=0" "$B" "$B backoff=0" "instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" > gpurun_out/r2v4_lat.jsonl 2> gpurun_out/r2v4_lat.err
PHASE_OPTS="instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" timeout 600 python tools/phase_trace.py 1024 1048576 > gpurun_out/r2v4_phase_i1.jsonl 2> gpurun_out/r2v4_phase_i1.err
tail -3 gpurun_out/r2v4_pytest.log gpurun_out/r2v4_pytest_mp.log; cat gpurun_out/r2v4_lat.jsonl; tail -3 gpurun_out/r2v4_lat.err
