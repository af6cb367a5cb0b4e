"""Reproduce one virtual-rank collective with option variants and report error / parity.
usage: python tools/repro.py algo coll n count kw="seed=0 fanout=2" opts1 ; opts2 ; ...
"""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import paper_conf_sigcomm_liuhlgcwz025_b200 as R
import resccl_inputs as inp
from oracle import ir as oir
from gpu_helpers import oracle_expect, run_virtual

algo, coll, n, count = sys.argv[1], sys.argv[2], int(sys.argv[3]), int(sys.argv[4])
kw = dict(x.split("=") for x in sys.argv[5].split()) if sys.argv[5] else {}
kw = {k: int(v) if v.isdigit() else v for k, v in kw.items()}
check = os.environ.get("REPRO_CHECK", "1") == "1"
for opts in " ".join(sys.argv[6:]).split(";"):
    g = oir.generate(algo, coll, n, **kw)
    for o in opts.split():
        k, v = o.split("=")
        g.extra[k] = v
    m = count * n if coll == "reducescatter" else count
    xs = inp.all_inputs("float32", 2, n, m)
    t = time.time()
    try:
        outs, info, err = run_virtual(R, g.to_text(), coll, xs, "float32", count)
    except Exception as e:
        print(opts, "EXC", e, flush=True)
        continue
    dt = time.time() - t
    ok = "skip"
    if check and err == 0:
        exp = oracle_expect(g, xs, "float32", count, chunk_bytes=int(g.extra.get("chunkbytes", 1 << 20)),
                            instances=int(g.extra.get("instances", 1)), K=int(g.extra.get("fifodepth", 4)))
        ok = all(np.array_equal(a.view(np.uint8), b.view(np.uint8)) for a, b in zip(outs, exp))
    print(opts, "err", err, "parity", ok, f"{dt:.1f}s", flush=True)
