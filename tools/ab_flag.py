"""A/B timing of an internal int switch of the library (e.g. dda__set_dyn_tail) on the default
block-Jacobi solve at 1M blocks, alternating settings in one process.  Tuning aid.
usage: python tools/ab_flag.py <setter> <v1,v2,...> [n] [reps]"""
import ctypes as C, os, sys, json, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
setter = sys.argv[1]
vals = [int(v) for v in sys.argv[2].split(",")]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 1_000_000
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 6
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
K.bj_setup()
f = getattr(dda.lib(), setter)
f.argtypes = [C.c_int]
res = {v: [] for v in vals}
its = {}
for r in range(reps + 1):
    for v in vals:
        f(v)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d, it, rr, st = K.pcg_solve(t["F"])
        b.record(); torch.cuda.synchronize()
        its[v] = (it, rr, st)
        if r:
            res[v].append(a.elapsed_time(b))
print(json.dumps({"setter": setter, "n": K.n, "median_ms": {v: statistics.median(res[v]) for v in vals},
                  "us_per_iter": {v: 1000 * statistics.median(res[v]) / its[v][0] for v in vals},
                  "all": res, "iters_rel_status": its}), flush=True)
