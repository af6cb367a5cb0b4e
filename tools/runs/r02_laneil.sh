# warp-interleaved lanes (leaders on different sub-partitions): same-box A/B and parity
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
M="instances=18 linkmodel=port chunkbytes=8388608 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[16777216, 33554432, 268435456]" timeout 1200 python tools/lat_graph.py "$M nwarps=8" "$M nwarps=8 laneil=1" "$M nwarps=4" "$M nwarps=4 laneil=1" "$M nwarps=16" "$M nwarps=16 laneil=1" > gpurun_out/lat_laneil.jsonl 2>&1
R="instances=14 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[1024, 16777216, 268435456]" timeout 900 python tools/lat_graph.py "$R nwarps=8" "$R nwarps=8 laneil=1" >> gpurun_out/lat_laneil.jsonl 2>&1
H="instances=4 chunkbytes=524288 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="[1048576, 4194304, 268435456]" timeout 900 python tools/lat_graph.py "$H nwarps=8" "$H nwarps=8 laneil=1" >> gpurun_out/lat_laneil.jsonl 2>&1
RESCCL_LANE_IL=1 timeout 1500 python -m pytest tests/test_gpu_engine_variants.py tests/test_gpu_parity.py tests/test_gpu_parity_r2.py tests/test_gpu_multiprocess.py -m gpu -x -q > gpurun_out/pytest_laneil.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_laneil.log
tail -n 2 gpurun_out/pytest_laneil.log
