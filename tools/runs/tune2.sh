mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0"
run() { echo "$* => $(timeout 120 $B "$@" 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])' 2>&1)"; }
{
for cb in 1048576 2097152 4194304; do for k in 2 3; do run --instances 16 --chunk-bytes $cb --fifo-depth $k; done; done
for cb in 1048576 2097152; do for k in 2 3; do run --instances 32 --nwarps 8 --chunk-bytes $cb --fifo-depth $k; done; done
run --instances 36 --nwarps 8 --chunk-bytes 2097152 --fifo-depth 2
run --instances 18 --chunk-bytes 2097152 --fifo-depth 2
run --instances 12 --chunk-bytes 2097152 --fifo-depth 2
run --instances 16 --chunk-bytes 1048576 --fifo-depth 2 --dtype float32
run --instances 16 --chunk-bytes 1048576 --fifo-depth 2 --size-mb 1024
run --instances 16 --chunk-bytes 1048576 --fifo-depth 2 --size-mb 64
} > gpurun_out/tune2.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --instances 16 --chunk-bytes 1048576 --fifo-depth 2 > gpurun_out/ncu_launch_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --instances 16 --chunk-bytes 1048576 --fifo-depth 2 > gpurun_out/ncu_full.log 2>&1
