mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python tools/sweep.py c2 > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
timeout 600 python tools/sweep.py c3 > gpurun_out/sweep_c3.jsonl 2> gpurun_out/sweep_c3.err
timeout 600 python tools/sweep.py c4 > gpurun_out/sweep_c4.jsonl 2> gpurun_out/sweep_c4.err
timeout 600 python tools/sweep.py f2 > gpurun_out/sweep_f2.jsonl 2> gpurun_out/sweep_f2.err
python bench.py --steps 20 --warmup 5 --sweep 1,16,64,1024 > gpurun_out/bench_r01_v3.json 2> gpurun_out/bench_r01_v3.err
