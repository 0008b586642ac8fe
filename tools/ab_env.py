"""A/B timing of environment switches of the library (read per solve, e.g. DDA_STRIP) on the default
block-Jacobi solve at 1M blocks, alternating settings in one process.  Tuning aid.
usage: python tools/ab_env.py "A=1,B=2;A=0" [n] [reps]"""
import os, sys, json, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
sets = [dict(kv.split("=") for kv in s.split(",") if kv) for s in sys.argv[1].split(";")]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1_000_000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 6
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
K.bj_setup()
keys = sorted({k for s in sets for k in s})
res = {i: [] for i in range(len(sets))}
its, dref, diff = {}, None, {}
for r in range(reps + 1):
    for i, s in enumerate(sets):
        for k in keys:
            os.environ.pop(k, None)
        os.environ.update(s)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d, it, rr, st = K.pcg_solve(t["F"])
        b.record(); torch.cuda.synchronize()
        its[i] = (it, rr, st)
        if dref is None:
            dref = d.clone()
        diff[i] = float((d - dref).abs().max() / dref.abs().max())
        if r:
            res[i].append(a.elapsed_time(b))
print(json.dumps({"n": K.n, "sets": sets, "median_ms": [statistics.median(res[i]) for i in res],
                  "us_per_iter": [1000 * statistics.median(res[i]) / max(its[i][0], 1) for i in res],
                  "iters_rel_status": [its[i] for i in res], "max_rel_diff_vs_first": [diff[i] for i in res],
                  "all": [res[i] for i in res]}), flush=True)
