"""Per-iteration cost of the partitioned solver (dda_pcg_solve_dist) with the loopback transport on
one GPU.  v5 / v4 / v3 run the partitions' kernels one after another, so their time is the driver's
overhead + the partitions' summed work; v6 runs every partition in one persistent kernel; v7 one persistent kernel per partition, concurrently.  Not a
scaling measurement.  DDA_DIST_CHUNK selects the host-check chunk."""
import json, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
if os.environ.get("DDA_LIB_PATH"):          # A/B against another build of the library
    dda.LIB_PATH = os.environ["DDA_LIB_PATH"]
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
out = {}
for nparts in (1, 2, 4):
    b = dda.row_bounds(P.n, nparts)
    comm = dda.Comm.loopback(nparts)
    t = dda.problem_to_device(P)
    Fs, keep = [], []
    for r in range(nparts):
        r0, r1 = int(b[r]), int(b[r + 1])
        K = comm.build_matrix_dist(r, P.n, b, t["kdiag"][r0:r1].contiguous(), t["bi"], t["bj"], t["pen"], t["e"],
                                   t["g"])
        keep.append(K)
        Fs.append(t["F"][6 * r0: 6 * r1].contiguous())
    for ver in ("7", "6", "5", "4", "4s", "3"):
        os.environ["DDA_DIST_VERSION"] = ver[0]
        os.environ["DDA_DIST_OVERLAP"] = "0" if ver == "4s" else "1"
        ms = []
        for rep in range(4):
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            ds, it, rr, st = comm.pcg_solve(Fs)
            e.record(); torch.cuda.synchronize()
            if rep: ms.append(a.elapsed_time(e))
        out[f"P{nparts}_v{ver}"] = {"iters": it, "rel_res": rr, "status": st, "ms": statistics.median(ms),
                                    "us_per_iter": 1000 * statistics.median(ms) / it}
    comm.free()
# the single-GPU scaled engine on the same system, for reference
Kg = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
Kg.pcg_solve(t["F"])
a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(); _, it1, _, _ = Kg.pcg_solve(t["F"]); e.record(); torch.cuda.synchronize()
out["single_gpu"] = {"iters": it1, "ms": a.elapsed_time(e), "us_per_iter": 1000 * a.elapsed_time(e) / it1}
print(json.dumps({"n": P.n, "chunk": os.environ.get("DDA_DIST_CHUNK", "8"), "loopback": out}), flush=True)
