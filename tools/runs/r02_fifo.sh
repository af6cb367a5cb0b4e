# launch / handoff floors and micro-batch x FIFO-depth sweep at mid sizes (device clock)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_robustness.py tests/test_nccl_shim.py tests/test_nvls.py tests/test_rescclang.py tests/test_timeline.py -m gpu -q > gpurun_out/pytest_gpu_tail.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_tail.log
export RESCCL_TIMEOUT_MS=20000
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/launch_floor tools/launch_floor.cu
for g in "96 384 224 14" "96 384 224 8" "96 384 0 14" "144 256 192 14" "16 384 224 14"; do timeout 60 /tmp/launch_floor $g; done > gpurun_out/launch_floor.jsonl 2>&1
O=""
for cb in 524288 1048576 2097152; do for k in 2 4 8; do O="$O|instances=14 nwarps=8 chunkbytes=$cb fifodepth=$k direct=1"; done; done
IFS='|' read -ra OPTS <<< "${O#|}"
LAT_SIZES="[4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "${OPTS[@]}" > gpurun_out/lat_fifo_ring.jsonl 2>&1
O=""
for cb in 1048576 2097152 4194304; do for k in 2 4 8; do O="$O|instances=18 nwarps=8 linkmodel=port chunkbytes=$cb fifodepth=$k direct=1"; done; done
IFS='|' read -ra OPTS <<< "${O#|}"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "${OPTS[@]}" > gpurun_out/lat_fifo_mesh.jsonl 2>&1
cat gpurun_out/launch_floor.jsonl; tail -3 gpurun_out/lat_fifo_ring.jsonl gpurun_out/lat_fifo_mesh.jsonl
