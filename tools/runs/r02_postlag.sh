# deferred post (postlag): micro-batch cost at mid sizes, ring and mesh (device clock)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=""
for cb in 1048576 2097152 4194304 33554432; do for pl in 0 1 2 4; do O="$O|instances=14 nwarps=8 chunkbytes=$cb fifodepth=2 direct=1 postlag=$pl"; done; done
IFS='|' read -ra OPTS <<< "${O#|}"
LAT_SIZES="[16777216, 67108864, 268435456]" timeout 1200 python tools/lat_graph.py "${OPTS[@]}" > gpurun_out/lat_postlag_ring.jsonl 2>&1
O=""
for cb in 1048576 2097152 4194304; do for pl in 0 2; do O="$O|instances=18 nwarps=8 linkmodel=port chunkbytes=$cb fifodepth=2 direct=1 postlag=$pl"; done; done
IFS='|' read -ra OPTS <<< "${O#|}"
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[4194304, 16777216, 67108864]" timeout 900 python tools/lat_graph.py "${OPTS[@]}" > gpurun_out/lat_postlag_mesh.jsonl 2>&1
RESCCL_POST_LAG=2 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_postlag2.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_postlag2.log
tail -n 3 gpurun_out/pytest_postlag2.log
