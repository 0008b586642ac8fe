"""Profiling driver: launches the PCG loop-body kernels directly (outside the CUDA graph,
whose conditional-node kernels ncu cannot profile individually) via dda__time_pcg_phases_ex.
Usage under ncu: -k regex:k_g_spmv|k_s_update --launch-skip 2 --launch-count 1."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
scaled = int(sys.argv[2]) if len(sys.argv) > 2 else 1
P = make_slope(preset(n, seed=1005))
t = dda.problem_to_device(P)
K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
L = dda.lib()
L.dda__time_pcg_phases_ex.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p, C.c_int]
d = torch.empty_like(t["F"])
ms = (C.c_float * 2)()
rc = L.dda__time_pcg_phases_ex(K.handle, C.c_void_p(t["F"].data_ptr()), C.c_void_p(d.data_ptr()), 5, ms, scaled)
print("rc", rc, "spmv ms", ms[0], "update ms", ms[1])
