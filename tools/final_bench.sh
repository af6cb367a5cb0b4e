mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
python bench.py --direct 0 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench_staged.json 2> gpurun_out/bench_staged.err
timeout 900 python tools/sweep.py c2 > gpurun_out/sweep_c2_direct.jsonl 2>&1
