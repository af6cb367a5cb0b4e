mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_engine_variants.py -m gpu -q -k small_cta > gpurun_out/pytest_small.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_small.log
LAT_ALGO=hm LAT_GOPTS=g=8 LAT_SIZES="[1024, 16384, 65536, 262144, 1048576]" timeout 600 python tools/lat_graph.py "instances=1 nwarps=2 chunkbytes=33554432 direct=1" "instances=1 nwarps=4 chunkbytes=33554432 direct=1" > gpurun_out/lat_small3.jsonl 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_small.json 2> gpurun_out/bench_small.err
tail -n 2 gpurun_out/pytest_small.log; cut -c1-160 gpurun_out/lat_small3.jsonl; python -c "import json; d=json.load(open('gpurun_out/bench_small.json')); print(d['value'], d['tuned_us'])"
