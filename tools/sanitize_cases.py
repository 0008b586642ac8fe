"""Workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

Runs every kernel family of the hot path once on a small system, through the C ABI:
assembly + value-only re-assembly, the symmetric SpMV (and full storage), the
block-Jacobi setup, PCG with each engine — the scaled persistent kernel k_sp_loop
(including its exact stopping test, phase C) and the single-reduction k_sp_cg1, the scaled graph loop, the unscaled
graph loop, the scaled SSOR-AI persistent kernel k_sp_ssor, the ILU(0) sync-free
sweeps — the partitioned solver over the loopback transport (P = 2), and contact
detection.  Every result is checked against the oracle's iteration count so a
sanitizer-perturbed schedule that changed a decision would show.

usage: compute-sanitizer --tool memcheck python tools/sanitize_cases.py [tiny|paper] [case ...]
"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import oracle
import paper_conf_ipps_xiaohmxw17_b200 as dda
from synth import make_slope, preset, random_vector


def engine(eng, loop):
    f = dda.lib().dda__set_pcg_engine
    f.argtypes = [ctypes.c_int]
    f(eng)
    g = dda.lib().dda__set_scaled_loop
    g.argtypes = [ctypes.c_int]
    g(loop)


CASES = ("build", "spmv", "bj_graph_phases", "bj_scaled_persistent", "bj_scaled_2phase", "bj_scaled_cg1", "bj_scaled_graph", "bj_graph", "bj_persistent", "ssor_ai",
         "ilu0", "none", "dist", "contacts")


def main(name, cases):
    torch.cuda.set_device(0)
    P = make_slope(preset(name))
    O = oracle.assemble(P)
    t = dda.problem_to_device(P)
    F = t["F"]
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    out = {}
    _, ito, _, _ = O.pcg(P.F, tol=1e-10, precond="bj")
    engines = {"bj_scaled_persistent": (2, 1), "bj_scaled_2phase": (2, 1), "bj_scaled_cg1": (2, 1),
               "bj_scaled_graph": (0 + 2, 0), "bj_graph": (0, -1), "bj_persistent": (1, -1)}
    forced = {"bj_scaled_2phase": "0", "bj_scaled_cg1": "1"}   # k_sp_loop / k_sp_cg1 (DDA_SCALED_CG1)
    for c in cases:
        print(f"case {c} ...", flush=True)
        if c == "build":
            K.update_values(t["kdiag"], t["pen"], t["e"], t["g"])
            K.bj_setup(full=True)
            out[c] = K.nnzb
        elif c == "spmv":
            x = torch.from_numpy(random_vector(P.n, 3)).cuda()
            y, yf = K.spmv(x), K.spmv_full(x)
            assert torch.allclose(y, yf, rtol=1e-12, atol=1e-9)
            out[c] = float(y.norm())
        elif c == "bj_graph_phases":
            # the unscaled graph engine's loop-body kernels launched directly (not from the graph)
            engine(0, -1)
            f = dda.lib().dda__time_pcg_phases
            f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
            d = torch.empty_like(F)
            ms = (ctypes.c_float * 2)()
            r = f(K.handle, ctypes.c_void_p(F.data_ptr()), ctypes.c_void_p(d.data_ptr()), -4, ms)
            engine(-1, -1)
            assert r == 0, r
            out[c] = (ms[0], ms[1])
        elif c in engines:
            engine(*engines[c])
            if c in forced:
                os.environ["DDA_SCALED_CG1"] = forced[c]
            d, it, rr, st = K.pcg_solve(F, tol=1e-10, precond="bj")
            os.environ.pop("DDA_SCALED_CG1", None)
            engine(-1, -1)
            out[c] = (it, st, K.last_checks())
            assert st == dda.OK and abs(it - ito) <= max(2, ito // 100), (c, it, ito)
        elif c in ("ssor_ai", "ilu0", "none"):
            _, itp, _, _ = O.pcg(P.F, tol=1e-10, precond=c)
            d, it, rr, st = K.pcg_solve(F, tol=1e-10, precond=c)
            K.precond_apply(F, precond=c)
            out[c] = (it, st, K.pcg_engine(c))
            assert st == dda.OK and abs(it - itp) <= max(2, itp // 100), (c, it, itp)
        elif c == "dist":
            # partitioned solver, loopback transport, 2 partitions built on the device (v3, then v2)
            b = dda.row_bounds(P.n, 2)
            comm = dda.Comm.loopback(2)
            Ks, Fs = [], []
            for r in range(2):
                r0, r1 = int(b[r]), int(b[r + 1])
                Ks.append(comm.build_matrix_dist(r, P.n, b, t["kdiag"][r0:r1].contiguous(), t["bi"], t["bj"],
                                                 t["pen"], t["e"], t["g"]))
                Fs.append(t["F"][6 * r0:6 * r1].contiguous())
            for v in ("1", "0"):
                os.environ["DDA_DIST_SCALED"] = v
                ds, it, rr, st = comm.pcg_solve(Fs, tol=1e-10, precond="bj")
                out[f"dist_v{3 if v == '1' else 2}"] = (it, st)
                assert st == dda.OK and abs(it - ito) <= max(2, ito // 100), ("dist", v, it, ito)
            os.environ.pop("DDA_DIST_SCALED")
            comm.spmv([torch.from_numpy(random_vector(int(b[r + 1] - b[r]), 5)).cuda() for r in range(2)])
            comm.free()
        elif c == "contacts":
            vptr = np.arange(0, 4 * P.n + 1, 4, dtype=np.int32)
            vxy = np.ascontiguousarray(P.verts.reshape(-1, 2))
            C = dda.detect_contacts(torch.from_numpy(vptr).cuda(), torch.from_numpy(vxy).cuda(), 0.2)
            C.springs(torch.from_numpy(np.ascontiguousarray(P.centroid)).cuda())
            out[c] = C.count
        else:
            raise SystemExit(f"unknown case {c}")
        torch.cuda.synchronize()
        print(f"case {c} ok: {out.get(c, '')}", flush=True)
    print(f"sanitize_cases {name}: n={P.n} oracle_bj_iters={ito} {out} ok", flush=True)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "tiny", sys.argv[2:] or CASES)
