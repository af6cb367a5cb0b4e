# lane leader state in shared memory: per-primitive setup gap, latency curve, parity
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
for ls in 0 1; do
  PHASE_RAW=gpurun_out/phase_raw_ls$ls.jsonl PHASE_OPTS="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1 lanesmem=$ls" timeout 300 python tools/phase_trace.py 1024 16777216 >> gpurun_out/phase_ls.jsonl 2>&1
done
B="instances=12 nwarps=12 tmatile=28672 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[1024, 1048576, 16777216, 67108864, 268435456]" timeout 900 python tools/lat_graph.py "$B" "$B lanesmem=1" "instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1 lanesmem=1" > gpurun_out/lat_ls.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1024, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1" "instances=18 nwarps=8 linkmodel=port chunkbytes=4194304 direct=1 lanesmem=1" "instances=1 nwarps=8 chunkbytes=33554432 direct=1" "instances=1 nwarps=8 chunkbytes=33554432 direct=1 lanesmem=1" >> gpurun_out/lat_ls.jsonl 2>&1
RESCCL_LANE_SMEM=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_r2.py -m gpu -x -q > gpurun_out/pytest_ls.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_ls.log
cat gpurun_out/lat_ls.jsonl; tail -n 2 gpurun_out/pytest_ls.log
