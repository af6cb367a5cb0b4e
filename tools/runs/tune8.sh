mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 900 python -m pytest tests -m gpu -x -q --timeout 200 > gpurun_out/gpu_tests8.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests8.log
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
run
run --direct 1
run --direct 1 --fifo-depth 4
run --direct 1 --chunk-bytes 2097152
run --direct 1 --chunk-bytes 8388608
run --direct 1 --instances 16
run --direct 1 --size-mb 1024
} > gpurun_out/tune8.txt 2>&1
