"""Times dda_build_matrix (A1) and dda_update_values at a given size (tuning aid)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
if os.environ.get("DDA_LIB_PATH"):          # A/B against another build of the library
    dda.LIB_PATH = os.environ["DDA_LIB_PATH"]
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
def ev(fn, reps=5):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn(); torch.cuda.synchronize(); a.record()
    for _ in range(reps): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps
build = ev(lambda: dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"]).free())
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
upd = ev(lambda: K.update_values(t["kdiag"], t["pen"], t["e"], t["g"]))
print(json.dumps({"n": K.n, "springs": P.m, "build_ms": build, "update_values_ms": upd}))
