"""Small-message latency probe: ring AR on 8 virtual ranks, bf16."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R
N = 8
OPTS = sys.argv[1:] or ["instances=18 chunkbytes=8388608 direct=1", "instances=18 chunkbytes=8388608 direct=1 backoff=0",
                        "instances=18 chunkbytes=8388608 direct=1 tma=0", "instances=18 chunkbytes=8388608 direct=1 tma=0 backoff=0",
                        "instances=2 chunkbytes=8388608 direct=1 tma=0 backoff=0", "instances=18 chunkbytes=4194304 direct=0"]
for opts in OPTS:
    text = R.rescclGenerateIr("ring", "allreduce", N)
    h, rest = text.split("\n", 1)
    grp = R.VirtualGroup(N, 0)
    grp.load(h + " " + opts + "\n" + rest)
    res = {}
    for S in [int(x) for x in os.environ.get('LAT_SIZES', str([1024, 65536, 1 << 20, 4 << 20, 16 << 20]))[1:-1].split(',')]:
        cnt = S // 2
        s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
        r = [torch.empty_like(x) for x in s]
        for _ in range(5): grp.allreduce(s, r)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10): grp.allreduce(s, r)
        e1.record(); torch.cuda.synchronize()
        res[S] = round(e0.elapsed_time(e1) / 10 * 1e3, 1)
    # empty kernel-ish baseline: count=1
    print(json.dumps({"opts": opts, "us": res}), flush=True)
    grp.destroy()
