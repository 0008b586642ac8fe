"""Host-side wall-clock breakdown of one bench step (where the GPU may sit idle)."""
import os, sys, time, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
rows = []
for rep in range(6):
    torch.cuda.synchronize()
    T = [time.perf_counter()]
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"]); torch.cuda.synchronize()
    T.append(time.perf_counter())
    K.bj_setup(); torch.cuda.synchronize()
    T.append(time.perf_counter())
    d, it, rr, st = K.pcg_solve(t["F"], tol=1e-10, maxit=10000); torch.cuda.synchronize()
    T.append(time.perf_counter())
    d, it, rr, st = K.pcg_solve(t["F"], tol=1e-10, maxit=10000); torch.cuda.synchronize()
    T.append(time.perf_counter())
    K.free(); torch.cuda.synchronize()
    T.append(time.perf_counter())
    rows.append([1e3 * (b - a) for a, b in zip(T, T[1:])])
for name, k in zip(["build", "bj_setup", "solve (first on K)", "solve (second on K)", "free"], range(5)):
    print(f"{name:22s} median {statistics.median(r[k] for r in rows[2:]):8.3f} ms")
