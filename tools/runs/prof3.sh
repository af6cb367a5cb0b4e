mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python bench.py > gpurun_out/bench_r01_v4.json 2> gpurun_out/bench_r01_v4.err
B="python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 0"
for cb in 4194304 16777216 33554432; do
  echo "chunk $cb => $($B --chunk-bytes $cb 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["frac"])')" >> gpurun_out/chunk_v4.txt
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v4.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v4 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v4.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_v4.ncu-rep --page raw --csv > gpurun_out/prof_v4_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_v4.ncu-rep --page details --csv > gpurun_out/prof_v4_details.csv 2>/dev/null
