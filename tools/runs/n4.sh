mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python - > gpurun_out/n4.jsonl 2>gpurun_out/n4.err <<'PY'
import sys, json
sys.path.insert(0, "tools"); sys.argv = ["sweep.py", "none"]
import sweep
for inst, nw, cb in [(37, 8, 32 << 20), (36, 8, 32 << 20), (32, 8, 32 << 20), (37, 16, 32 << 20), (37, 8, 64 << 20), (37, 8, 16 << 20)]:
    d = sweep.measure("ring", "allreduce", "", dict(instances=inst, chunkbytes=cb, fifodepth=2, nwarps=nw, direct=1), 1 << 30, iters=10, n=4)
    d["nwarps"] = nw; d["chunkbytes"] = cb
    print(json.dumps(d), flush=True)
PY
cat gpurun_out/n4.jsonl | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['instances'], d['nwarps'], d['chunkbytes']>>20, d['busbw_gbs'], d['err'])"
tail -2 gpurun_out/n4.err
