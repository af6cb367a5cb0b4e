mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 900 python -m pytest tests -m gpu -x -q --timeout 200 > gpurun_out/gpu_tests5.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests5.log
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
run
run --tma 0
for tile in 8192 16384; do for st in 2 3 4 6; do RESCCL_TMA_TILE=$tile RESCCL_TMA_STAGES=$st run; done; done
for inst in 8 12 16 18; do for cb in 1048576 2097152 4194304; do run --instances $inst --chunk-bytes $cb; done; done
run --fifo-depth 3
run --fifo-depth 4
} > gpurun_out/tune4.txt 2>&1
