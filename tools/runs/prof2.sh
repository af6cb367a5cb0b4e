mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r01_v2.json 2> gpurun_out/bench_r01_v2.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v2.log 2>&1
