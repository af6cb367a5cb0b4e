mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000
python - > gpurun_out/warps_c3c4.jsonl 2>&1 <<'PY'
import json, sys, os
sys.path.insert(0, os.getcwd())
sys.argv = ["sweep"]
import importlib.util
spec = importlib.util.spec_from_file_location("sw", "tools/sweep.py")
PY
for w in 4 6 8; do
  SW_NW=$w python - >> gpurun_out/warps_c3c4.jsonl 2>&1 <<'PY'
import os, sys, json
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tools"))
sys.argv = ["sweep.py", "none"]
import sweep as S
w = int(os.environ["SW_NW"])
for name, g, o in (("dbt", "", dict(chunkbytes=8 << 20, fifodepth=2, tbbudget=16, linkmodel="port", direct=1)),
                   ("hm", "g=4", dict(chunkbytes=1 << 20, fifodepth=2, tbbudget=16, direct=1))):
    o = dict(o, nwarps=w)
    S.emit(S.measure(name, "allreduce", g, o, 256 << 20))
for coll, cb in (("allgather", 8 << 20), ("reducescatter", 2 << 20)):
    S.emit(S.measure("synth", coll, "seed=0 fanout=2", dict(instances=4, chunkbytes=cb, fifodepth=2, nwarps=w, direct=1), 256 << 20))
PY
done
