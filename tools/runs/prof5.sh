mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v5.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v5 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v5.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_v5.ncu-rep --page raw --csv > gpurun_out/prof_v5_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_v5.ncu-rep --page details --csv > gpurun_out/prof_v5_details.csv 2>/dev/null
