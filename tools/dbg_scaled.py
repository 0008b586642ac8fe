"""Debug: scaled BJ engine arrays and iterates vs numpy / the oracle."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_xiaohmxw17_b200 as dda
import oracle
from synth import make_slope, preset
name = sys.argv[1] if len(sys.argv) > 1 else "tiny"
P = make_slope(preset(name) if not name.isdigit() else preset(int(name), seed=1005))
O = oracle.assemble(P)
S = O.export()
K = dda.build_from_problem(P)
L = dda.lib()
L.dda__scaled_export.argtypes = [C.c_void_p] * 4
n, z = K.n, K.nnzb
su = np.zeros((z, 36)); lf = np.zeros((n, 24)); sf = np.zeros((n, 24))
print("export rc", L.dda__scaled_export(K.handle, su.ctypes.data, lf.ctypes.data, sf.ctypes.data))
def untile(b):
    A = np.zeros((6, 6))
    for q in range(9):
        R, Cc = divmod(q, 3)
        A[2*R, 2*Cc], A[2*R, 2*Cc+1], A[2*R+1, 2*Cc], A[2*R+1, 2*Cc+1] = b[4*q:4*q+4]
    return A
def unpack_lo(v):
    M = np.zeros((6, 6))
    for r in range(6):
        for c in range(r + 1):
            M[r, c] = v[r*(r+1)//2 + c]
    return M
Lr = np.linalg.cholesky(S.diag)
errL = max(np.abs(unpack_lo(lf[i]) - Lr[i]).max() / np.abs(Lr[i]).max() for i in range(n))
errS = max(np.abs(unpack_lo(sf[i]) - np.linalg.inv(Lr[i])).max() / np.abs(np.linalg.inv(Lr[i])).max() for i in range(n))
urow = np.repeat(np.arange(n), np.diff(S.row_ptr))
Si = np.linalg.inv(Lr)
errV = 0.0
for u in range(z):
    ref = Si[urow[u]] @ S.upper[u] @ Si[S.col_idx[u]].T
    errV = max(errV, np.abs(untile(su[u]) - ref).max() / max(np.abs(ref).max(), 1e-300))
print("errL", errL, "errS", errS, "errV", errV, flush=True)
F = torch.from_numpy(P.F).cuda()
f = L.dda__set_pcg_engine
f.argtypes = [C.c_int]
for eng in (0, 2):
    f(eng)
    for mi in (1, 2, 3, 12):
        d, it, rr, st = K.pcg_solve(F, tol=1e-300, maxit=mi)
        dm, itm, _, _ = O.pcg(P.F, tol=1e-300, maxit=mi, precond="bj")
        d = d.cpu().numpy()
        print(eng, mi, it, itm, np.linalg.norm(d - dm) / np.linalg.norm(dm), flush=True)
