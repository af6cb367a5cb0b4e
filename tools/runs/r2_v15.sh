mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python bench.py > gpurun_out/r2v15_bench.json 2> gpurun_out/r2v15_bench.err
cat gpurun_out/r2v15_bench.json; tail -3 gpurun_out/r2v15_bench.err
