"""Device timeline of the persistent scaled PCG loop (k_sp_loop) via %globaltimer stamps
(internal hook dda__set_loop_trace).  Prints per-phase work / barrier times (us).  Tuning aid."""
import ctypes as C, os, sys, json, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
K.bj_setup()
L = dda.lib()
L.dda__set_pcg_engine.argtypes = [C.c_int]
L.dda__set_scaled_loop.argtypes = [C.c_int]
L.dda__set_loop_trace.argtypes = [C.c_void_p, C.c_void_p, C.c_int]
L.dda__set_pcg_engine(2)
L.dda__set_scaled_loop(1)
d, it, rr, st = K.pcg_solve(t["F"])
G = L.dda__set_loop_trace(K.handle, None, 0)
iters = it + 2
buf = torch.zeros((iters + 1) * G * 4, dtype=torch.int64, device="cuda")
L.dda__set_loop_trace(K.handle, C.c_void_p(buf.data_ptr()), iters)
ms_plain = []
for _ in range(3):
    L.dda__set_loop_trace(K.handle, None, 0)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); K.pcg_solve(t["F"]); b.record(); torch.cuda.synchronize()
    ms_plain.append(a.elapsed_time(b))
L.dda__set_loop_trace(K.handle, C.c_void_p(buf.data_ptr()), iters)
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
d, it, rr, st = K.pcg_solve(t["F"])
b.record(); torch.cuda.synchronize()
L.dda__set_loop_trace(K.handle, None, 0)
Tall = buf.cpu().numpy().reshape(iters + 1, G, 4).astype(np.float64) / 1000.0   # us
T = Tall[:it]
kernel_us = Tall[iters, 0, 1] - Tall[iters, 0, 0]
loop_us = T[it - 1, 0, 3] - T[0, 0, 0]
ks = range(1, it - 1)
A = [np.median(T[k, :, 1] - T[k, :, 0]) for k in ks]
Amax = [np.max(T[k, :, 1]) - np.min(T[k, :, 0]) for k in ks]
bar1 = [np.median(T[k, :, 2] - T[k, :, 1]) for k in ks]
B = [np.median(T[k, :, 3] - T[k, :, 2]) for k in ks]
it_t = [T[k + 1, 0, 0] - T[k, 0, 0] for k in ks]
bar2 = [np.median(T[k + 1, :, 0] - T[k, :, 3]) for k in ks]
spread = [np.max(T[k, :, 1]) - np.min(T[k, :, 1]) for k in ks]
skew0 = [np.max(T[k, :, 0]) - np.min(T[k, :, 0]) for k in ks]
med = statistics.median
print(json.dumps({"ms_untraced": ms_plain, "kernel_ms": kernel_us / 1000, "loop_ms": loop_us / 1000,
                  "entry_to_first_iter_us": T[0, 0, 0] - Tall[iters, 0, 0], "n": K.n, "G": G, "iters": it, "rel": rr, "solve_ms": a.elapsed_time(b),
                  "iter_us": med(it_t), "phaseA_cta_median_us": med(A), "phaseA_span_us": med(Amax),
                  "phaseA_end_spread_us": med(spread), "start_skew_us": med(skew0),
                  "barrier1_median_wait_us": med(bar1), "phaseB_cta_median_us": med(B),
                  "barrier2_median_wait_us": med(bar2),
                  "iter_us_pct": [float(np.percentile(it_t, q)) for q in (10, 50, 90, 99)],
                  "iter_us_mean": float(np.mean(it_t)),
                  "first_iters_us": [float(x) for x in it_t[:6]],
                  "bar2_over_30us": [(int(k), float(b)) for k, b in zip(ks, bar2) if b > 30][:60],
                  "phaseA_by_decile": [float(np.mean(A[j * len(A) // 10:(j + 1) * len(A) // 10])) for j in range(10)]}),
      flush=True)
