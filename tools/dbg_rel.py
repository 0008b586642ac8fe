"""Debug: reported true residual vs an independent recomputation (K.spmv) over repeated bench-like steps."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
F = t["F"]
for rep in range(5):
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    K.bj_setup()
    d, it, rr, st = K.pcg_solve(F, tol=1e-10, maxit=10000)
    y = K.spmv(d)
    rel = float(torch.linalg.norm(F - y) / torch.linalg.norm(F))
    print(rep, K.pcg_engine(), it, rr, st, "recomputed", rel, "|d|", float(torch.linalg.norm(d)), flush=True)
    d2, it2, rr2, st2 = K.pcg_solve(F, tol=1e-10, maxit=10000)
    print("   second solve", it2, rr2, st2, float(torch.linalg.norm(d2 - d)), flush=True)
    K.free()
