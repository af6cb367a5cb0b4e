mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity_r2.py -q -x -m gpu -k "size_based" > gpurun_out/r2v13_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v13_pytest.log
tail -2 gpurun_out/r2v13_pytest.log
B="nwarps=8 fifodepth=2 direct=1"
SZ="[1024, 16384, 65536, 262144, 1048576, 4194304, 16777216, 67108864, 268435456]"
LAT_SIZES="$SZ" timeout 900 python tools/lat_graph.py "instances=14 chunkbytes=33554432 $B" "instances=18 chunkbytes=33554432 $B" > gpurun_out/r2v13_ring.jsonl 2> gpurun_out/r2v13.err
RESCCL_COOP=0 LAT_SIZES="[1024, 1048576, 16777216]" timeout 900 python tools/lat_graph.py "instances=14 chunkbytes=33554432 $B" > gpurun_out/r2v13_ring_nocoop.jsonl 2>> gpurun_out/r2v13.err
LAT_ALGO=hm LAT_GOPTS="g=8" LAT_SIZES="$SZ" timeout 1200 python tools/lat_graph.py "instances=1 chunkbytes=33554432 $B" "instances=2 chunkbytes=33554432 $B" "instances=4 chunkbytes=4194304 $B" "instances=18 chunkbytes=2097152 linkmodel=port $B" "instances=18 chunkbytes=33554432 linkmodel=port $B" "instances=14 chunkbytes=8388608 linkmodel=port $B" > gpurun_out/r2v13_mesh.jsonl 2>> gpurun_out/r2v13.err
cat gpurun_out/r2v13_ring_nocoop.jsonl; tail -3 gpurun_out/r2v13.err
