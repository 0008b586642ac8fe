"""A/B of dda_spmv kernel paths selected by environment switches (e.g. DDA_SPMV_TMA=1) in one process:
bitwise comparison of y and CUDA-event time per SpMV (median of rounds of `reps` calls), reported as
algorithmic GB/s (392 + 300u bytes per block row) and fraction of the measured HBM peak.
usage: python tools/spmv_ab.py "DDA_SPMV_TMA=0;DDA_SPMV_TMA=1" [n] [reps]"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

sets = [dict(kv.split("=") for kv in s.split(",") if kv) for s in sys.argv[1].split(";")]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1_000_000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 20
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
x = torch.empty(6 * K.n, dtype=torch.float64, device="cuda").uniform_(-1, 1)
u = K.nnzb / K.n
bytes_ = K.n * (392 + 300 * u)
try:
    peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                       "MEASURED_PEAKS.json")))["hbm_gbs"]
except Exception:
    peak = None
keys = sorted({k for s in sets for k in s})
res = {i: [] for i in range(len(sets))}
ys = {}
for rnd in range(6):
    for i, s in enumerate(sets):
        for k in keys:
            os.environ.pop(k, None)
        os.environ.update(s)
        y = K.spmv(x)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(reps):
            K.spmv(x, y)
        b.record(); torch.cuda.synchronize()
        ys[i] = y
        if rnd:
            res[i].append(a.elapsed_time(b) / reps)
out = []
for i, s in enumerate(sets):
    ms = statistics.median(res[i])
    gbs = bytes_ / (ms * 1e-3) / 1e9
    out.append({"set": s, "ms": ms, "gbs": gbs, "frac": gbs / peak if peak else None,
                "bit_identical_to_first": bool(torch.equal(ys[i], ys[0]))})
print(json.dumps({"n": K.n, "u": u, "peak_gbs": peak, "results": out}), flush=True)
