mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for inst in 4 8 16 18; do for cb in 262144 1048576; do for k in 2 4 8; do
  echo "inst=$inst cb=$cb k=$k $(timeout 120 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 --instances $inst --chunk-bytes $cb --fifo-depth $k 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])' 2>&1)"
done; done; done > gpurun_out/tune1.txt 2>&1
