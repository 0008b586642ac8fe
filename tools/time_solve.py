"""Times repeated dda_pcg_solve calls on one matrix (tuning aid; env knobs select variants)."""
import os, sys, json, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
K.bj_setup()
ms = []
for r in range(reps + 2):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    d, it, rr, st = K.pcg_solve(t["F"])
    b.record(); torch.cuda.synchronize()
    if r >= 2:
        ms.append(a.elapsed_time(b))
env = {k: v for k, v in os.environ.items() if k.startswith("DDA_")}
print(json.dumps({"env": env, "n": K.n, "iters": it, "rel": rr, "ms_median": statistics.median(ms),
                  "us_per_iter": 1000 * statistics.median(ms) / it, "ms": ms}), flush=True)
