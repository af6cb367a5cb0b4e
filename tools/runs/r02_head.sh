mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_head.log 2>&1; echo "smoke=$?" >> gpurun_out/smoke_head.log
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_head.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_head.log
python bench.py > gpurun_out/bench_head.json 2> gpurun_out/bench_head.err
timeout 600 python tools/lat_graph.py > gpurun_out/lat_graph_head.jsonl 2>&1
tail -3 gpurun_out/smoke_head.log gpurun_out/pytest_gpu_head.log; head -c 800 gpurun_out/bench_head.json
