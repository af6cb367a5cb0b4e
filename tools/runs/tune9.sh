mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
run
run --chunk-bytes 16777216
run --chunk-bytes 33554432
for tile in 8192 16384; do for st in 3 4 6; do echo "tile $tile st $st"; RESCCL_TMA_TILE=$tile RESCCL_TMA_STAGES=$st run; done; done
run --instances 12
run --instances 9
run --nwarps 8 --instances 18
run --nwarps 12 --instances 18
RESCCL_L2HINT=0 run
} > gpurun_out/tune9.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_direct python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_direct.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_direct.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
