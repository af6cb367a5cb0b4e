# batched writable-credit lookahead: A/B on the tuned classes and the ring, phase timeline, parity
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
M="instances=18 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1"
M16="instances=16 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1"
R="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
H="instances=4 nwarps=8 chunkbytes=524288 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[4194304, 16777216, 33554432]" timeout 900 python tools/lat_graph.py "$M" "$M labatch=4" "$M labatch=8" "$M" > gpurun_out/lat_la.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[67108864, 268435456]" timeout 900 python tools/lat_graph.py "$M16" "$M16 labatch=4" >> gpurun_out/lat_la.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="[1048576, 4194304, 8388608]" timeout 900 python tools/lat_graph.py "$H" "$H labatch=4" >> gpurun_out/lat_la.jsonl 2>&1
LAT_SIZES="[16777216, 67108864, 268435456]" timeout 900 python tools/lat_graph.py "$R" "$R labatch=4" >> gpurun_out/lat_la.jsonl 2>&1
PHASE_ALGO=hm PHASE_GOPTS=g=8 PHASE_RAW=gpurun_out/phase_raw_la.jsonl PHASE_OPTS="$M labatch=4" timeout 300 python tools/phase_trace.py 16777216 > /dev/null 2>&1
RESCCL_LA_BATCH=4 timeout 1500 python -m pytest tests/test_gpu_engine_variants.py tests/test_gpu_parity.py tests/test_gpu_parity_r2.py tests/test_gpu_multiprocess.py -m gpu -x -q > gpurun_out/pytest_la.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_la.log
tail -n 2 gpurun_out/pytest_la.log
