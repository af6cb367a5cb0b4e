# one-sided fences (splitfence): latency curve A/B, phase timeline, parity
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
B="instances=12 nwarps=12 tmatile=28672 chunkbytes=33554432 fifodepth=2 direct=1"
R="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 67108864, 268435456]" timeout 900 python tools/lat_graph.py "$B splitfence=0" "$B" "$R splitfence=0" "$R" > gpurun_out/lat_sf.jsonl 2>&1
M="instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1024, 4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "$M splitfence=0" "$M" "instances=1 nwarps=8 chunkbytes=33554432 direct=1 splitfence=0" "instances=1 nwarps=8 chunkbytes=33554432 direct=1" >> gpurun_out/lat_sf.jsonl 2>&1
PHASE_RAW=gpurun_out/phase_raw_sf.jsonl PHASE_OPTS="$R" timeout 300 python tools/phase_trace.py 1024 16777216 > gpurun_out/phase_sf.jsonl 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py tests/test_gpu_fullsize.py tests/test_gpu_multiprocess.py -m gpu -x -q > gpurun_out/pytest_sf.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_sf.log
RESCCL_JITTER=1 timeout 600 python -m pytest tests/test_gpu_robustness.py -m gpu -x -q -k jitter > gpurun_out/pytest_sf_jitter.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_sf_jitter.log
cat gpurun_out/lat_sf.jsonl | cut -c1-220; tail -n 2 gpurun_out/pytest_sf.log gpurun_out/pytest_sf_jitter.log
