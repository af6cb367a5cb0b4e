mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
R="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
B="instances=12 nwarps=12 tmatile=28672 chunkbytes=33554432 fifodepth=2 direct=1"
M="instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1"
P="instances=1 nwarps=8 chunkbytes=33554432 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 67108864, 268435456]" timeout 900 python tools/lat_graph.py "$R" "$R prepnext=1" "$B" "$B prepnext=1" > gpurun_out/lat_pn.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1024, 4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "$M" "$M prepnext=1" "$P" "$P prepnext=1" >> gpurun_out/lat_pn.jsonl 2>&1
PHASE_RAW=gpurun_out/phase_raw_pn.jsonl PHASE_OPTS="$R prepnext=1" timeout 300 python tools/phase_trace.py 16777216 > /dev/null 2>&1
RESCCL_PREP_NEXT=1 timeout 1500 python -m pytest tests/test_gpu_engine_variants.py tests/test_gpu_parity.py tests/test_gpu_parity_r2.py -m gpu -x -q > gpurun_out/pytest_pn.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_pn.log
cut -c1-200 gpurun_out/lat_pn.jsonl; tail -n 2 gpurun_out/pytest_pn.log
