"""Fig. 10a analogue: ResCCL workflow phase times vs scale on the host.
The paper's Fig. 16 HM AllReduce program text is run at nNodes x 8 GPUs, 16..1024."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sigcomm_liuhlgcwz025_b200 as R
src = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden",
                        "fig16_hm_allreduce.py.txt")).read()
top = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
nn = 2
while nn * 8 <= top:
    s = src.replace("    nNodes = 4\n", f"    nNodes = {nn}\n").replace("nRanks =32", f"nRanks ={nn * 8}")
    t = time.time()
    p = R.rescclProfilePlanner(s, "", verify=True)  # the deadlock check runs at every scale (deadlock_free null = unchecked)
    p["wall_s"] = round(time.time() - t, 2)
    p["host_cores"] = os.cpu_count()
    print(json.dumps(p), flush=True)
    nn *= 2
