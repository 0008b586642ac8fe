"""NEXT-2: the paper's SpMV comparison re-run on B200 (HSBCSR 2.8x over cuSPARSE on the K40):
the paper's HSBCSR two-stage kernel (dda_hsbcsr_spmv), this build's single-pass symmetric kernel
(dda_spmv) and cuSPARSE's BSR SpMV on the full matrix (through torch's BSR tensor), on the
case-1-sized matrix (4361 + 18731 blocks) and slope matrices up to 1M blocks.  One JSON line each."""
import json, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import case1_like, make_slope, preset

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
try:
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6552.0)
except OSError:
    peak = 6552.0


def time_fn(fn, reps=30):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


cases = sys.argv[1].split(",") if len(sys.argv) > 1 else ["case1", "64000", "256000", "1000000"]
for c in cases:
    if c == "case1":
        n, kd, bi, bj, pen, e, g, F = case1_like()
    else:
        P = make_slope(preset(int(c), seed=1040))
        n, kd, bi, bj, pen, e, g = P.n, P.kdiag, P.bi, P.bj, P.pen, P.e, P.g
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    K = dda.build_matrix(dev(kd), dev(bi), dev(bj), dev(pen), dev(e), dev(g))
    H = dda.HSBCSR(K)
    ex = K.export()
    nnzb = K.nnzb
    rows = np.concatenate([np.arange(n), np.repeat(np.arange(n), np.diff(ex["row_ptr"])), ex["col_idx"]])
    cols = np.concatenate([np.arange(n), ex["col_idx"], np.repeat(np.arange(n), np.diff(ex["row_ptr"]))])
    vals = np.concatenate([ex["diag"], ex["upper"], np.transpose(ex["upper"], (0, 2, 1))])
    order = np.lexsort((cols, rows))
    crow = np.zeros(n + 1, np.int64)
    np.add.at(crow, rows[order] + 1, 1)
    A = torch.sparse_bsr_tensor(torch.from_numpy(np.cumsum(crow)).cuda(),
                                torch.from_numpy(cols[order].astype(np.int64)).cuda(),
                                torch.from_numpy(np.ascontiguousarray(vals[order])).cuda(), size=(6 * n, 6 * n))
    x = torch.rand(6 * n, dtype=torch.float64, device="cuda") * 2 - 1
    y1, y2 = torch.empty_like(x), torch.empty_like(x)
    K.spmv(x, y1)
    H.spmv(x, y2)
    yc = A @ x
    t_sym = time_fn(lambda: K.spmv(x, y1))
    t_hs = time_fn(lambda: H.spmv(x, y2))
    t_cs = time_fn(lambda: A @ x)
    u = nnzb / n
    b_sym = n * (392 + 300 * u)                                   # algorithmic bytes, single pass
    print(json.dumps({
        "case": c, "blocks": n, "offdiag_blocks": nnzb, "u": round(u, 3),
        "dda_spmv_us": 1000 * t_sym, "hsbcsr_us": 1000 * t_hs, "cusparse_full_bsr_us": 1000 * t_cs,
        "hsbcsr_over_cusparse": t_cs / t_hs, "dda_spmv_over_hsbcsr": t_hs / t_sym,
        "dda_spmv_over_cusparse": t_cs / t_sym,
        "dda_spmv_frac_hbm": b_sym / (t_sym * 1e-3) / 1e9 / peak,
        "hsbcsr_bytes_per_row": 392 + 300 * u + 2 * 96 * u + 0,   # + up-res / low-res written and read back
        "rel_diff_hs": float(torch.linalg.norm(y2 - y1) / torch.linalg.norm(y1)),
        "rel_diff_cusparse": float(torch.linalg.norm(yc - y1) / torch.linalg.norm(y1)),
        "paper": "HSBCSR 2.8x over cuSPARSE on the K40, case 1 (P:222)"}), flush=True)
    del A, H, K
    torch.cuda.empty_cache()
