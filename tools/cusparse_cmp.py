"""configs[3] / Z23: the paper's SpMV comparison on B200 — the symmetric BSR6 kernel (dda_spmv, upper
storage only) against cuSPARSE's BSR SpMV on the FULL matrix (both triangles; "recover the
global stiffness matrix", "2.8x over cuSPARSE"), reached through torch's sparse BSR tensor
(torch dispatches BSR @ vector on CUDA to cuSPARSE).  Library call used as the comparison baseline
only.  One JSON line per size."""
import json, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

sizes = [int(s) for s in (sys.argv[1] if len(sys.argv) > 1 else "64000,256000,1000000").split(",")]
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json"))).get("hbm_gbs", 6552.0) \
    if os.path.exists(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")) else 6552.0


def time_fn(fn, reps=20):
    fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


for n_req in sizes:
    P = make_slope(preset(n_req, seed=1040))
    t = dda.problem_to_device(P)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    ex = K.export()
    n, nnzb = K.n, K.nnzb
    # full block CSR: diagonal + upper + lower (transposed upper), rows sorted by column
    rows = np.concatenate([np.arange(n), np.repeat(np.arange(n), np.diff(ex["row_ptr"])), ex["col_idx"]])
    cols = np.concatenate([np.arange(n), ex["col_idx"], np.repeat(np.arange(n), np.diff(ex["row_ptr"]))])
    vals = np.concatenate([ex["diag"], ex["upper"], np.transpose(ex["upper"], (0, 2, 1))])
    order = np.lexsort((cols, rows))
    rows, cols, vals = rows[order], cols[order], np.ascontiguousarray(vals[order])
    crow = np.zeros(n + 1, np.int64)
    np.add.at(crow, rows + 1, 1)
    crow = np.cumsum(crow)
    A = torch.sparse_bsr_tensor(torch.from_numpy(crow).cuda(), torch.from_numpy(cols.astype(np.int64)).cuda(),
                                torch.from_numpy(vals).cuda(), size=(6 * n, 6 * n))
    x = torch.rand(6 * n, dtype=torch.float64, device="cuda") * 2 - 1
    y = torch.empty_like(x)
    # correctness of the comparison: cuSPARSE full product == symmetric product (rounding)
    yc = A @ x
    K.spmv(x, y)
    rel = float(torch.linalg.norm(yc - y) / torch.linalg.norm(y))
    t_sym = time_fn(lambda: K.spmv(x, y))
    t_cs = time_fn(lambda: A @ x)
    u = nnzb / n
    b_sym = n * (392 + 300 * u)
    b_full = n * (392 + 584 * u)
    print(json.dumps({"blocks": n, "u": round(u, 3), "sym_ms": t_sym, "cusparse_full_bsr_ms": t_cs,
                      "speedup_sym_over_cusparse": t_cs / t_sym, "rel_diff": rel,
                      "sym_gbs": b_sym / (t_sym * 1e-3) / 1e9, "sym_frac": b_sym / (t_sym * 1e-3) / 1e9 / peak,
                      "cusparse_gbs_full_bytes": b_full / (t_cs * 1e-3) / 1e9,
                      "cusparse_frac": b_full / (t_cs * 1e-3) / 1e9 / peak,
                      "paper": "2.8x over cuSPARSE on the K40 (P:222)"}), flush=True)
    del A, K
    torch.cuda.empty_cache()
