mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 600 python -m pytest tests -m gpu -x -q --timeout 120 > gpurun_out/gpu_tests3.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests3.log
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])' 2>/dev/null || tail -3 gpurun_out/last_err.txt)"; }
{
run --tma 0
run --tma 1
for tile in 8192 16384 32768; do for st in 2 4; do RESCCL_TMA_TILE=$tile RESCCL_TMA_STAGES=$st run --tma 1; done; done
run --tma 1 --instances 18
run --tma 1 --chunk-bytes 1048576
run --tma 1 --chunk-bytes 4194304
run --tma 1 --fifo-depth 3
run --tma 1 --instances 32 --nwarps 8
run --tma 0 --instances 32 --nwarps 8
} > gpurun_out/tune3.txt 2>&1
