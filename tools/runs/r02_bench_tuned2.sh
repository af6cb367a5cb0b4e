mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python bench.py > gpurun_out/bench_tuned2.json 2> gpurun_out/bench_tuned2.err
python -c "import json; d=json.load(open('gpurun_out/bench_tuned2.json')); print(d['value'], d['roofline']['frac'], d['tuned_busbw_gbs'], d['tuned_us'])"
