mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 900 python -m pytest tests -m gpu -x -q --timeout 200 > gpurun_out/gpu_tests6.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests6.log
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>gpurun_out/last_err.txt | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["async_error"])' 2>/dev/null || tail -2 gpurun_out/last_err.txt)"; }
{
run
for tile in 8192 12288; do for st in 2 3 4; do echo "tile=$tile st=$st"; RESCCL_TMA_TILE=$tile RESCCL_TMA_STAGES=$st run; done; done
RESCCL_TMA_TILE=6144 RESCCL_TMA_STAGES=8 run
run --tma 0
} > gpurun_out/tune5.txt 2>&1
timeout 300 python tools/tb_util.py 64 > gpurun_out/tb_util.jsonl 2> gpurun_out/tb_util.err
