mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python tools/sweep.py nr > gpurun_out/sweep_nr.jsonl 2> gpurun_out/sweep_nr.err
tail -3 gpurun_out/sweep_nr.err
cat gpurun_out/sweep_nr.jsonl | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['nranks'], d['bytes']>>20, 'MiB', d['busbw_gbs'], d['blocks'], d['err'])"
