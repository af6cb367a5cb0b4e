export RESCCL_TIMEOUT_MS=10000
timeout 500 python tools/lat.py "instances=18 chunkbytes=8388608 direct=1" "instances=18 chunkbytes=8388608 direct=1 tmamin=262144" "instances=18 chunkbytes=8388608 direct=1 tmamin=131072" "instances=18 chunkbytes=4194304 direct=0" > gpurun_out/lat3.jsonl 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q --timeout 200 -k "edge or config1 or direct_edge or monotone" > gpurun_out/gpu_tests9.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests9.log
