mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multiprocess.py -q -x -m gpu -k "graph or direct" > gpurun_out/r2v25_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v25_pytest.log
tail -2 gpurun_out/r2v25_pytest.log
B="nwarps=8 fifodepth=2 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 268435456]" timeout 600 python tools/lat_graph.py "instances=14 chunkbytes=33554432 $B" > gpurun_out/r2v25_lat.jsonl 2> gpurun_out/r2v25.err
LAT_ALGO=hm LAT_GOPTS="g=8" LAT_SIZES="[1024, 65536, 262144]" timeout 600 python tools/lat_graph.py "instances=1 chunkbytes=2097152 $B" "instances=2 chunkbytes=2097152 $B" >> gpurun_out/r2v25_lat.jsonl 2>> gpurun_out/r2v25.err
cat gpurun_out/r2v25_lat.jsonl | cut -c1-200
