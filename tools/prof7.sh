# HEAD capture: multicast probe, launch list + ncu --set full of the bench kernel, SM-budget sweep
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 120 python tools/probe_multicast.py > gpurun_out/probe_multicast.json 2>&1
nvidia-smi topo -m > gpurun_out/topo.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v7.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v7 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v7.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_v7.ncu-rep --page raw --csv > gpurun_out/prof_v7_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_v7.ncu-rep --page details --csv > gpurun_out/prof_v7_details.csv 2>/dev/null
rm -f gpurun_out/prof_ring_ar8_v7.ncu-rep
timeout 600 python tools/sm_budget.py 256 two > gpurun_out/sm_budget_v7.jsonl 2>&1
