mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python bench.py > gpurun_out/bench_r01_v6.json 2> gpurun_out/bench_r01_v6.err
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all_v6.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v6.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v6 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v6.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_v6.ncu-rep --page raw --csv > gpurun_out/prof_v6_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_v6.ncu-rep --page details --csv > gpurun_out/prof_v6_details.csv 2>/dev/null
