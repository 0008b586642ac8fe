"""Times the PCG loop-body kernels individually (internal hook dda__time_pcg_phases)."""
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
L.dda__time_pcg_phases_ex.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p, C.c_int]
d = torch.empty_like(t["F"])
u = K.nnzb / K.n
for scaled in (0, 1):
    ms = (C.c_float * 2)()
    rc = L.dda__time_pcg_phases_ex(K.handle, C.c_void_p(t["F"].data_ptr()), C.c_void_p(d.data_ptr()), 20, ms,
                                   scaled)
    # algorithmic bytes per row: unscaled SpMV + 96 / update 528; scaled SpMV
    # without D (300u + 8 + 192) + deferred x update (96) / update 144 (r~, q~ read; r~ written)
    spmv_bytes = K.n * ((300 * u + 296) if scaled else (392 + 300 * u + 96))
    upd_bytes = K.n * (144 if scaled else 528)
    print(json.dumps({"scaled": scaled, "rc": rc, "n": K.n, "spmv_fused_ms": ms[0],
                      "spmv_fused_gbs": spmv_bytes / ms[0] / 1e6,
                      "update_ms": ms[1], "update_gbs": upd_bytes / ms[1] / 1e6}))
