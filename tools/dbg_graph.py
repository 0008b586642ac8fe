import sys, ctypes; sys.path.insert(0,'/root/repo')
import torch, numpy as np
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset
f = dda.lib().dda__set_pcg_engine; f.argtypes=[ctypes.c_int]; f(0)
for name,cfg in [("ragged_1k", preset(1000, seed=1041)), ("tiny", preset("tiny")), ("paper", preset("paper"))]:
    P = make_slope(cfg)
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    L = dda.lib()
    import ctypes as C
    it, rr = C.c_int32(), C.c_double()
    d = torch.empty_like(F)
    st = L.dda_pcg_solve(K.handle, C.c_void_p(F.data_ptr()), None, C.c_void_p(d.data_ptr()), 1e-10, 10000, 1, 1.0, C.byref(it), C.byref(rr), None)
    print(name, P.n, "status", st, L.dda_status_string(st), L.dda_last_cuda_error(), it.value, rr.value, flush=True)
