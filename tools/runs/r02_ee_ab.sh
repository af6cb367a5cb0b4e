# early loop exit A/B on one box: bench geometry and the 14-instance ring, interleaved
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
B="instances=12 nwarps=12 tmatile=28672 chunkbytes=33554432 fifodepth=2 direct=1"
R="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
LAT_SIZES="[16777216, 67108864, 268435456]" timeout 1200 python tools/lat_graph.py "$B earlyexit=0" "$B earlyexit=1" "$B earlyexit=0" "$B earlyexit=1" "$R earlyexit=0" "$R earlyexit=1" > gpurun_out/lat_ee_ab.jsonl 2>&1
for e in 0 1 0 1; do RESCCL_EARLY_EXIT=$e python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 0 --tuned-sweep "" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('earlyexit', $e, d['value'], d['ms_per_step'])"; done > gpurun_out/bench_ee_ab.txt 2>&1
cat gpurun_out/bench_ee_ab.txt
# size classes for the tuned selection: HM 2x4 (pair) against the mesh at 1-16 MiB
LAT_ALGO=hm LAT_GOPTS=g=4 LAT_SIZES="[1048576, 2097152, 4194304, 8388608, 16777216]" timeout 900 python tools/lat_graph.py "instances=2 nwarps=8 chunkbytes=1048576 direct=1" "instances=4 nwarps=8 chunkbytes=524288 direct=1" "instances=4 nwarps=8 chunkbytes=1048576 direct=1" "instances=4 nwarps=8 chunkbytes=2097152 direct=1" > gpurun_out/lat_classes.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1048576, 2097152, 4194304, 8388608, 16777216]" timeout 900 python tools/lat_graph.py "instances=2 nwarps=8 chunkbytes=2097152 direct=1" "instances=18 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1" >> gpurun_out/lat_classes.jsonl 2>&1
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[67108864, 268435456]" timeout 900 python tools/lat_graph.py "instances=14 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1" "instances=16 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1" >> gpurun_out/lat_classes.jsonl 2>&1
