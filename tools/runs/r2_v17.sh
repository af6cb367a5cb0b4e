mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 1200 python -m pytest tests/test_gpu_parity_r2.py tests/test_gpu_multiprocess.py -q -m gpu -k "pushreduce or registered" > gpurun_out/r2v17_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v17_pytest.log
tail -3 gpurun_out/r2v17_pytest.log
B="instances=14 chunkbytes=33554432 nwarps=8 fifodepth=2 direct=1"
LAT_SIZES="[1048576, 16777216, 268435456]" timeout 600 python tools/lat_graph.py "$B" "$B pushreduce=1" > gpurun_out/r2v17_lat.jsonl 2> gpurun_out/r2v17_lat.err
cat gpurun_out/r2v17_lat.jsonl
