mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python - > gpurun_out/inst128.jsonl 2>gpurun_out/inst128.err <<'PY'
import sys, json
sys.path.insert(0, "tools"); sys.argv = ["sweep.py", "none"]
import sweep
for n, inst in [(4, 28), (4, 30), (4, 32), (8, 14), (8, 15), (8, 16), (8, 17), (8, 18)]:
    for S in (256 << 20, 1 << 30):
        d = sweep.measure("ring", "allreduce", "", dict(instances=inst, chunkbytes=32 << 20, fifodepth=2, nwarps=8, direct=1), S, iters=10, n=n)
        print(json.dumps(d), flush=True)
PY
cat gpurun_out/inst128.jsonl | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['nranks'], d['instances'], d['blocks'], d['bytes']>>20, d['busbw_gbs'], d['err'])"
for i in 16 18; do timeout 300 python bench.py --instances $i --nwarps 8 --chunk-bytes 33554432 --no-cpu-baseline --e2e-steps 0 --sweep "" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench inst=$i', d['value'], d['config']['inplace_busbw_gbs'], d['config']['blocks_total'])"; done
