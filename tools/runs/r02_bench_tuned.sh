mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python bench.py > gpurun_out/bench_tuned.json 2> gpurun_out/bench_tuned.err
tail -3 gpurun_out/bench_tuned.err; python -c "import json; d=json.load(open('gpurun_out/bench_tuned.json')); print(d['value'], d['roofline']['frac'], d['tuned_busbw_gbs'], d['tuned_us'], d['tuned_schedules'])"
