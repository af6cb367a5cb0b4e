mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
run
RESCCL_L2HINT=0 run
run --fifo-depth 3
run --fifo-depth 4
run --chunk-bytes 4194304
run --chunk-bytes 4194304 --fifo-depth 3
run --instances 18
run --instances 18 --chunk-bytes 4194304
run --size-mb 64
run --size-mb 1024
} > gpurun_out/tune6.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q --timeout 200 > gpurun_out/gpu_tests7.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests7.log
ncu --set full --clock-control none -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v3 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v3.log 2>&1
