mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
run
RESCCL_TMA_STAGES=2 run --nwarps 8 --instances 36
RESCCL_TMA_STAGES=2 RESCCL_TMA_TILE=16384 run --nwarps 8 --instances 36
RESCCL_TMA_STAGES=3 RESCCL_TMA_TILE=8192 run --nwarps 8 --instances 36
RESCCL_TMA_STAGES=2 run --nwarps 8 --instances 32
RESCCL_TMA_STAGES=2 run --nwarps 12 --instances 36
} > gpurun_out/tune11.txt 2>&1
SWEEP_DIRECT=1 timeout 900 python tools/sweep.py c3 c4 f2 > gpurun_out/sweep_c34_direct.jsonl 2>&1
