mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python tools/probe_multicast.py > gpurun_out/probe_multicast.json 2>&1
nvidia-smi topo -m > gpurun_out/topo.txt 2>&1
timeout 900 python tools/sm_budget.py 256 two one > gpurun_out/sm_budget.jsonl 2> gpurun_out/sm_budget.err
LAT_SIZES="[1024,65536,1048576,4194304,16777216]" timeout 300 python tools/lat.py "instances=37 nwarps=8 tmastages=2 tmatile=12288 chunkbytes=33554432 direct=1" "instances=1 chunkbytes=33554432 direct=1" "instances=4 chunkbytes=33554432 direct=1" > gpurun_out/lat.jsonl 2>&1
cat gpurun_out/probe_multicast.json gpurun_out/sm_budget.jsonl gpurun_out/lat.jsonl
