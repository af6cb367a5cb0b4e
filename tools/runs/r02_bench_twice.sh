mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
for i in 1 2; do python bench.py --no-cpu-baseline --e2e-steps 0 --tuned-sweep "" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks'])"; done
nvidia-smi --query-gpu=name,clocks.mem,clocks.max.mem,power.draw,temperature.gpu --format=csv
