"""configs[3]: SpMV bandwidth sweep 1k-4M blocks, symmetric BSR6 (dda_spmv) vs
full-storage BSR6 (dda_spmv_full), course-major and shuffled ordering, hot
(back-to-back, as PCG sees it) and cold (L2 flushed by a 512 MB write between
launches).  Algorithmic bytes per block row: symmetric 392 + 300u,
full 392 + 584u.  Prints one JSON line per point."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

PEAK = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"]


def timeit(fn, reps, flush=None):
    """Device time per launch.  The launches are captured in a CUDA graph and
    replayed, so host (Python / ctypes) overhead is not measured.  Hot:
    `reps` launches back to back.  Cold: each launch preceded by a 512 MB write
    (timed separately and subtracted)."""
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()

    def graph_of(body):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            body()
        return g

    def timed(g, n):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g.replay(); torch.cuda.synchronize()
        ts = []
        for _ in range(n):
            a.record(); g.replay(); b.record(); torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ts.sort()
        return ts[len(ts) // 2]

    if flush is None:
        g = graph_of(lambda: [fn() for _ in range(reps)])
        t = timed(g, 5) / reps
        return t, t
    gf = graph_of(lambda: [flush.add_(1.0) for _ in range(reps)])
    gb = graph_of(lambda: [(flush.add_(1.0), fn()) for _ in range(reps)])
    t = (timed(gb, 5) - timed(gf, 5)) / reps
    return t, t


def main():
    sizes = [int(s) for s in (sys.argv[1] if len(sys.argv) > 1 else "1000,4000,16000,64000,256000,1000000,4000000").split(",")]
    shuf = os.environ.get("SHUFFLE_AT", "16000,256000,1000000").split(",")
    flush = torch.zeros(64 * 1024 * 1024, dtype=torch.float64, device="cuda")    # 512 MB > L2
    import numpy as np
    for t, n in enumerate(sizes):
        for sh in (["course", "shuffled", "shuffled+rcm"] if str(n) in shuf else ["course"]):
            P = make_slope(preset(n, seed=1040 + t, shuffle=(sh != "course")))
            if sh == "shuffled+rcm":                       # NEXT-2: dda_rcm_order renumbering
                perm = dda.rcm_order(P.n, P.bi, P.bj)
                P.kdiag, P.bi, P.bj, P.F = dda.renumber(perm, P.kdiag, P.bi, P.bj, P.F)
            K = dda.build_from_problem(P)
            u = K.nnzb / K.n
            x = torch.rand(6 * K.n, dtype=torch.float64, device="cuda") * 2 - 1
            y = torch.empty_like(x)
            reps = 50 if K.n <= 300_000 else 20
            out = {"blocks": K.n, "nnzb_upper": K.nnzb, "u": round(u, 3), "order": sh, "shuffled": sh != "course"}
            for name, fn, bpr in (("sym", lambda: K.spmv(x, y), 392 + 300 * u),
                                  ("full", lambda: K.spmv_full(x, y), 392 + 584 * u)):
                hot_med, hot_min = timeit(fn, reps)
                cold_med, cold_min = timeit(fn, max(5, reps // 4), flush)
                by = K.n * bpr
                out[name] = {"hot_ms": hot_med, "cold_ms": cold_med, "bytes": by,
                             "hot_gbs": by / hot_med / 1e6, "cold_gbs": by / cold_med / 1e6,
                             "hot_frac": by / hot_med / 1e6 / PEAK, "cold_frac": by / cold_med / 1e6 / PEAK,
                             "gflops_hot": K.n * (72 + 144 * u) / hot_med / 1e6}
            out["full_over_sym_time_hot"] = out["full"]["hot_ms"] / out["sym"]["hot_ms"]
            out["l2_resident"] = K.n * (392 + 300 * u) < 2 * 126e6
            print(json.dumps(out), flush=True)
            K.free()
            del x, y


if __name__ == "__main__":
    main()
