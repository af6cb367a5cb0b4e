"""Small collectives on virtual ranks of cuda:0, checked against the oracle; used under
compute-sanitizer (memcheck / synccheck / racecheck) and with RESCCL_JITTER=1."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import paper_conf_sigcomm_liuhlgcwz025_b200 as R
import resccl_inputs as inp
from oracle import ir as oir
from gpu_helpers import oracle_expect, run_virtual

big = os.environ.get("SMALL_RUN_TMA") == "1"
cases = [("ring", "allreduce", 2, {}), ("hm", "allreduce", 8, {"g": 4}), ("ring", "allgather", 4, {}),
         ("synth", "reducescatter", 4, {"seed": 1, "fanout": 2}), ("dbt", "allreduce", 4, {})]
bad = 0
for name, coll, n, kw in cases:
    for direct in (0, 1):
        g = oir.generate(name, coll, n, **kw)
        count = (3 << 20) // 4 + 5 if big else 3000
        g.extra.update(chunkbytes=str(1 << 20 if big else 2048), instances="2", fifodepth="2", direct=str(direct))
        if big:
            g.extra["tmamin"] = "1024"
        m = count * n if coll == "reducescatter" else count
        xs = inp.all_inputs("float32", 2, n, m)
        outs, info, err = run_virtual(R, g.to_text(), coll, xs, "float32", count)
        exp = oracle_expect(g, xs, "float32", count, chunk_bytes=int(g.extra["chunkbytes"]), instances=2, K=2)
        ok = err == 0 and all(np.array_equal(a.view(np.uint8), b.view(np.uint8)) for a, b in zip(outs, exp))
        print(name, coll, n, "direct" if direct else "staged", "OK" if ok else "MISMATCH", flush=True)
        bad += not ok
print("ALL OK" if bad == 0 else f"{bad} FAILED")
sys.exit(1 if bad else 0)
