mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
for pf in 0 1 2 4; do echo "prefetch=$pf"; RESCCL_PREFETCH=$pf run; RESCCL_PREFETCH=$pf run --instances 18 --chunk-bytes 4194304; done
run --instances 18 --chunk-bytes 4194304 --fifo-depth 3
run --instances 18 --chunk-bytes 2097152 --fifo-depth 3
RESCCL_TMA_TILE=16384 RESCCL_TMA_STAGES=3 run --instances 18 --chunk-bytes 4194304
} > gpurun_out/tune7.txt 2>&1
