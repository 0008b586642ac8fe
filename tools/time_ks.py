"""Experiment: bare off-diagonal Ks products (one gathered vector; read-only vs coherent loads; 3 vs 4
CTAs/SM) against the fused scaled-engine SpMV (internal hook dda__time_ks_variants)."""
import ctypes as C, os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
L = dda.lib()
L.dda__time_ks_variants.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p]
d = torch.empty_like(t["F"])
ms = (C.c_float * 5)()
rc = L.dda__time_ks_variants(K.handle, C.c_void_p(t["F"].data_ptr()), C.c_void_p(d.data_ptr()), 10, ms)
u = K.nnzb / K.n
b_bare = K.n * (300 * u + 8 + 96)
print(json.dumps({"rc": rc, "n": K.n, "bare_ldg_3": ms[0], "bare_coherent_3": ms[1], "bare_ldg_4": ms[2],
                  "bare_coherent_4": ms[3], "fused_scaled": ms[4],
                  "bare_ldg_3_gbs": b_bare / (ms[0] * 1e-3) / 1e9}))
