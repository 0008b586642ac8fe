"""A/B timing of the scaled engine's two loop drivers (persistent cooperative kernel vs CUDA-graph
while loop) in one process, alternating, on one matrix.  Tuning aid."""
import ctypes as C, os, sys, json, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 6
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
K.bj_setup()
L = dda.lib()
L.dda__set_pcg_engine.argtypes = [C.c_int]
L.dda__set_scaled_loop.argtypes = [C.c_int]
L.dda__set_pcg_engine(2)
loops = [int(v) for v in (sys.argv[3].split(",") if len(sys.argv) > 3 else ["0", "1"])]
res = {l: [] for l in loops}
its = {}
for r in range(reps + 1):
    for loop in loops:
        L.dda__set_scaled_loop(loop)
        K.pcg_solve(t["F"])          # (re)build the engine for this loop kind
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d, it, rr, st = K.pcg_solve(t["F"])
        b.record(); torch.cuda.synchronize()
        its[loop] = (it, rr, K.last_checks())
        if r:
            res[loop].append(a.elapsed_time(b))
names = {0: "graph", 1: "persistent"}
print(json.dumps({"n": K.n, **{names[l] + "_ms": statistics.median(res[l]) for l in loops},
                  **{names[l] + "_all": res[l] for l in loops}, "iters_rel_checks": its}), flush=True)
