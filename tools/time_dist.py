"""Per-iteration cost of the partitioned solver (dda_pcg_solve_dist) with the loopback transport on
one GPU: P partitions run one after another, so this is the driver's overhead + the partitions'
summed work, not a scaling measurement.  DDA_DIST_CHUNK selects the host-check chunk."""
import json, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
if os.environ.get("DDA_LIB_PATH"):          # A/B against another build of the library
    dda.LIB_PATH = os.environ["DDA_LIB_PATH"]
from paper_conf_ipps_xiaohmxw17_b200.partition import row_bounds, local_from_slope
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
out = {}
for nparts in (1, 2):
    b = row_bounds(P.n, nparts)
    comm = dda.Comm.loopback(nparts)
    Fs, keep = [], []
    for r in range(nparts):
        lp = local_from_slope(P, b, r)
        K = dda.build_local(lp)
        comm.attach(r, K, lp)
        keep.append((K, lp))
        Fs.append(torch.from_numpy(P.F[6 * lp.r0: 6 * lp.r1].copy()).cuda())
    ms = []
    for rep in range(4):
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        ds, it, rr, st = comm.pcg_solve(Fs)
        e.record(); torch.cuda.synchronize()
        if rep: ms.append(a.elapsed_time(e))
    out[nparts] = {"iters": it, "rel_res": rr, "status": st, "ms": statistics.median(ms),
                   "us_per_iter": 1000 * statistics.median(ms) / it}
    comm.free()
print(json.dumps({"n": P.n, "chunk": os.environ.get("DDA_DIST_CHUNK", "8"), "loopback": out}), flush=True)
