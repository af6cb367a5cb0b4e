mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multiprocess.py -q -x -m gpu -k "graph or direct or registered" > gpurun_out/r2v12_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v12_pytest.log
tail -2 gpurun_out/r2v12_pytest.log
B="nwarps=8 fifodepth=2 direct=1"
LAT_SIZES="[1024, 65536, 1048576, 16777216, 67108864]" timeout 600 python tools/lat_graph.py "instances=14 chunkbytes=33554432 $B" > gpurun_out/r2v12_lat_ring.jsonl 2> gpurun_out/r2v12_lat.err
LAT_ALGO=hm LAT_GOPTS="g=8" LAT_SIZES="[1024, 65536, 1048576, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "instances=1 chunkbytes=33554432 $B" "instances=2 chunkbytes=33554432 $B" "instances=1 chunkbytes=33554432 linkmodel=port $B" "instances=14 chunkbytes=33554432 linkmodel=port $B" "instances=18 chunkbytes=2097152 linkmodel=port $B" > gpurun_out/r2v12_lat_mesh.jsonl 2>> gpurun_out/r2v12_lat.err
cat gpurun_out/r2v12_lat_ring.jsonl gpurun_out/r2v12_lat_mesh.jsonl; tail -3 gpurun_out/r2v12_lat.err
