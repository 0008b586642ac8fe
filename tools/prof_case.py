"""Profiling driver: one problem, a few SpMV launches and one short PCG launch.
Used under ncu (see profiles/README.md).  Not a benchmark."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

ap = argparse.ArgumentParser()
ap.add_argument("--blocks", type=int, default=1_000_000)
ap.add_argument("--spmv", type=int, default=3)
ap.add_argument("--pcg-maxit", type=int, default=20)
ap.add_argument("--precond", default="bj")
ap.add_argument("--shuffle", action="store_true")
a = ap.parse_args()
P = make_slope(preset(a.blocks, seed=1005, shuffle=a.shuffle))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
x = torch.rand(6 * K.n, dtype=torch.float64, device="cuda")
y = torch.empty_like(x)
for _ in range(a.spmv):
    K.spmv(x, y)
K.bj_setup()
d, it, rr, st = K.pcg_solve(t["F"], maxit=a.pcg_maxit, precond=a.precond)
torch.cuda.synchronize()
print("n", K.n, "nnzb", K.nnzb, "iters", it, "status", st)
