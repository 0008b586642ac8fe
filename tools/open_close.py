"""NEXT-1 measurement: the DDA open-close inner loop around the solve.

Within one time step the contact list is fixed; each open-close iteration changes the spring
penalties and states (a contact that opens drops its springs: penalty 0; lock <-> slide changes
the shear spring), the matrix VALUES are rebuilt ("rebuilt in every loop") and K d = F is
re-solved warm-started from the previous iteration's d.  This times, on the configs[4]
1M-block slope:
  cold   dda_build_matrix + dda_bj_setup + dda_pcg_solve(d0 = 0)            (the bench step)
  loop   dda_update_values (cached structure and sort permutations) + dda_bj_setup +
         dda_pcg_solve(d0 = previous d), for `loops` perturbations of the penalties
Perturbation per loop (seeded): every penalty x (1 + 0.02 U(-1,1)); 1% of the springs open (p = 0).
The structure is unchanged (p = 0 keeps the block, reading Z10), so value-only re-assembly applies.
Tuning/measurement aid; prints one JSON line."""
import json, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
loops = int(sys.argv[2]) if len(sys.argv) > 2 else 6
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
rng = np.random.default_rng(77)


def ev():
    e = torch.cuda.Event(enable_timing=True)
    e.record()
    return e


for _ in range(2):                                          # warm-up (allocator, engine build)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    K.bj_setup()
    K.pcg_solve(t["F"])
    K.free()
torch.cuda.synchronize()
e0 = ev()
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
e1 = ev()
K.bj_setup()
e2 = ev()
d, it0, rr0, st0 = K.pcg_solve(t["F"])
e3 = ev()
torch.cuda.synchronize()
cold = {"build_ms": e0.elapsed_time(e1), "bj_ms": e1.elapsed_time(e2), "solve_ms": e2.elapsed_time(e3),
        "iters": it0, "rel_res": rr0}
pen0 = P.pen.copy()
rows = []
dbuf = [torch.empty_like(t["F"]), torch.empty_like(t["F"])]    # ping-pong: d0 and d must differ per loop
dcold = torch.empty_like(t["F"])
for k in range(loops):
    pen = pen0 * (1.0 + 0.02 * rng.uniform(-1.0, 1.0, size=pen0.shape))
    pen[rng.random(pen0.shape[0]) < 0.01] = 0.0
    pen_d = torch.from_numpy(pen).cuda()
    torch.cuda.synchronize()
    a = ev()
    K.update_values(t["kdiag"], pen_d, t["e"], t["g"])
    b = ev()
    K.bj_setup()
    c = ev()
    # the result buffers are allocated before the timed call: a first-time torch allocation inside it
    # (cudaMalloc through the caching allocator) cost ~50 ms of host time in round 1's first loop
    dw, itw, rrw, stw = K.pcg_solve(t["F"], d0=d, d=dbuf[k % 2])
    e = ev()
    torch.cuda.synchronize()
    # the same system cold, for the iteration saving of the warm start
    _, itc, _, _ = K.pcg_solve(t["F"], d=dcold)
    assert stw == dda.OK and rrw <= 1.01e-10, (stw, rrw)
    rows.append({"update_values_ms": a.elapsed_time(b), "bj_ms": b.elapsed_time(c), "solve_ms": c.elapsed_time(e),
                 "iters_warm": itw, "iters_cold": itc, "rel_res": rrw})
    d = dw
med = lambda key: statistics.median(r[key] for r in rows)
print(json.dumps({"n": K.n, "springs": int(P.pen.shape[0]), "cold_step": cold, "loops": rows,
                  "median_loop": {k: med(k) for k in ("update_values_ms", "bj_ms", "solve_ms", "iters_warm",
                                                      "iters_cold")},
                  "loop_ms_median": statistics.median(r["update_values_ms"] + r["bj_ms"] + r["solve_ms"] for r in rows),
                  "cold_step_ms": cold["build_ms"] + cold["bj_ms"] + cold["solve_ms"]}), flush=True)
