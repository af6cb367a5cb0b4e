# grouped dependency-free pull-send posts: mesh / ring latency A/B, phase timeline, parity
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
M="instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1024, 65536, 1048576, 4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "$M postgroup=0" "$M" "instances=1 nwarps=8 chunkbytes=33554432 direct=1 postgroup=0" "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=2 nwarps=8 chunkbytes=33554432 direct=1" > gpurun_out/lat_pg.jsonl 2>&1
PHASE_ALGO=hm PHASE_GOPTS=g=8 PHASE_RAW=gpurun_out/phase_raw_mesh_pg.jsonl PHASE_OPTS="$M" timeout 300 python tools/phase_trace.py 1024 16777216 > gpurun_out/phase_mesh_pg.jsonl 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py tests/test_gpu_fullsize.py tests/test_gpu_multiprocess.py tests/test_gpu_api_rules.py -m gpu -x -q > gpurun_out/pytest_pg.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_pg.log
cut -c1-200 gpurun_out/lat_pg.jsonl; tail -n 2 gpurun_out/pytest_pg.log
