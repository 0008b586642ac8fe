"""ORACLE — TEST INFRASTRUCTURE ONLY.

ctypes front-end for `oracle/oracle.c`, the plain single-threaded CPU
implementation of what the hot path computes.
Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline /
`--impl reference` legs may import this package.  It shares no code with the
CUDA path in `paper_conf_ipps_xiaohmxw17_b200/` and never imports it.

Every function here is pinned in tests/test_oracle_*.py against something
other than itself (library routines, closed forms, brute force, special
cases).  Parity unpinned: none of these functions (the paper's printed timings
are context only).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OK, ERR_ARG, ERR_OOM, ERR_NOT_SPD, ERR_BREAKDOWN, ERR_NO_CONVERGENCE = 0, 1, 3, 4, 5, 6
PC = {"none": 0, "bj": 1, "ssor_ai": 2, "ilu0": 3}


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (no FMA contraction: values round as written)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-fPIC", "-shared", "-Wall", "-Wno-unused-label", "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        P = C.c_void_p
        L.orc_assemble.argtypes = [C.c_int32, P, C.c_int64, P, P, P, P, P, C.POINTER(C.c_void_p)]
        L.orc_assemble.restype = C.c_int
        L.orc_info.argtypes = [P, C.POINTER(C.c_int32), C.POINTER(C.c_int64)]
        L.orc_export.argtypes = [P] * 8
        L.orc_free.argtypes = [P]
        L.orc_expand.argtypes = [P]
        L.orc_full_nnz.argtypes = [P]
        L.orc_full_nnz.restype = C.c_int64
        L.orc_full_export.argtypes = [P, P, P, P]
        L.orc_spmv.argtypes = [P, P, P]
        L.orc_spmv_rows.argtypes = [P, P, C.c_int64, P, P]
        L.orc_spmv_par.argtypes = [P, P, P, C.POINTER(C.c_int32)]
        L.orc_bj_inv.argtypes = [P, P, C.POINTER(C.c_int32)]
        L.orc_ssor_ai_apply.argtypes = [P, P, C.c_double, P, P]
        L.orc_ilu0_factor.argtypes = [P]
        L.orc_ilu0_apply.argtypes = [P, P, P]
        L.orc_pcg.argtypes = [P, P, P, P, C.c_double, C.c_int32, C.c_int32, C.c_double,
                              C.POINTER(C.c_int32), C.POINTER(C.c_double), P]
        L.orc_ldlt_solve.argtypes = [P, P, P]
        L.orc_detect_contacts.argtypes = [C.c_int32, P, P, C.c_double, C.c_int32, C.c_int32, C.c_int64,
                                          P, P, P, P, P, P, P]
        L.orc_detect_contacts.restype = C.c_int64
        L.orc_contact_springs.argtypes = [C.c_int32, P, P, P, C.c_int64, P, P, P, P, P, P, C.c_double,
                                          C.c_double, P, P, P, P, P]
        L.orc_contact_springs.restype = C.c_int64
        L.orc_classify_contacts.argtypes = [C.c_int32, P, P, C.c_int64, P, P, P, P, P, C.c_double, P]
        L.orc_contact_transfer.argtypes = [C.c_int64, P, P, P, C.c_int64, P, P, P, P]
        L.orc_contact_transfer.restype = C.c_int64
        L.orc_contact_loads.argtypes = [C.c_int32, P, P, C.c_int64, P, P, P, P, P, P, P, P, P]
        L.orc_contact_check.argtypes = [C.c_int32, P, P, C.c_int64, P, P, P, P, P, P, P, P, C.c_double,
                                        C.c_double, C.c_double, C.c_double, P, P, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


class OracleError(RuntimeError):
    def __init__(self, code, what):
        super().__init__(f"oracle {what} failed with status {code}")
        self.code = code


@dataclass
class Structure:
    row_ptr: np.ndarray
    col_idx: np.ndarray
    low_ptr: np.ndarray
    low_row: np.ndarray
    low_to_up: np.ndarray
    diag: np.ndarray      # [n,6,6]
    upper: np.ndarray     # [nnzb,6,6]


class OracleMatrix:
    """O-1 assembled matrix (upper-symmetric BSR6) owned by the C oracle."""

    def __init__(self, n, kdiag, bi, bj, pen, e, g):
        L = lib()
        self._keep = [np.ascontiguousarray(kdiag, np.float64), np.ascontiguousarray(bi, np.int32),
                      np.ascontiguousarray(bj, np.int32), np.ascontiguousarray(pen, np.float64),
                      np.ascontiguousarray(e, np.float64), np.ascontiguousarray(g, np.float64)]
        kd, bi_, bj_, pen_, e_, g_ = self._keep
        h = C.c_void_p()
        st = L.orc_assemble(int(n), _p(kd), int(bi_.shape[0]), _p(bi_), _p(bj_), _p(pen_), _p(e_), _p(g_),
                            C.byref(h))
        self._keep = None
        if st != OK:
            raise OracleError(st, "assemble")
        self.h = h
        nn, nz = C.c_int32(), C.c_int64()
        L.orc_info(h, C.byref(nn), C.byref(nz))
        self.n, self.nnzb = int(nn.value), int(nz.value)

    @classmethod
    def from_problem(cls, P):
        return cls(P.n, P.kdiag, P.bi, P.bj, P.pen, P.e, P.g)

    def __del__(self):
        h = getattr(self, "h", None)
        if h is not None and _lib is not None:
            _lib.orc_free(h)
            self.h = None

    def export(self) -> Structure:
        n, z = self.n, self.nnzb
        s = Structure(np.empty(n + 1, np.int32), np.empty(z, np.int32), np.empty(n + 1, np.int32),
                      np.empty(z, np.int32), np.empty(z, np.int32), np.empty((n, 6, 6)), np.empty((z, 6, 6)))
        lib().orc_export(self.h, _p(s.row_ptr), _p(s.col_idx), _p(s.low_ptr), _p(s.low_row),
                         _p(s.low_to_up), _p(s.diag), _p(s.upper))
        return s

    def full_csr(self):
        """O-2 full scalar CSR as (indptr int64, indices int32, data float64)."""
        L = lib()
        nnz = L.orc_full_nnz(self.h)
        if nnz < 0:
            raise OracleError(ERR_OOM, "expand")
        ip = np.empty(6 * self.n + 1, np.int64); ix = np.empty(nnz, np.int32); dv = np.empty(nnz)
        L.orc_full_export(self.h, _p(ip), _p(ix), _p(dv))
        return ip, ix, dv

    def spmv(self, x):
        x = np.ascontiguousarray(x, np.float64)
        y = np.empty(6 * self.n)
        st = lib().orc_spmv(self.h, _p(x), _p(y))
        if st != OK:
            raise OracleError(st, "spmv")
        return y


    def spmv_par(self, x):
        """O-3 split over OpenMP threads (timing variant, bitwise equal to spmv).  Returns (y, threads)."""
        x = np.ascontiguousarray(x, np.float64)
        y = np.empty(6 * self.n)
        th = C.c_int32()
        st = lib().orc_spmv_par(self.h, _p(x), _p(y), C.byref(th))
        if st != OK:
            raise OracleError(st, "spmv_par")
        return y, int(th.value)
    def spmv_rows(self, rows, x):
        rows = np.ascontiguousarray(rows, np.int64)
        x = np.ascontiguousarray(x, np.float64)
        y = np.empty(rows.shape[0])
        lib().orc_spmv_rows(self.h, _p(rows), int(rows.shape[0]), _p(x), _p(y))
        return y

    def bj_inv(self):
        dinv = np.empty((self.n, 6, 6))
        bad = C.c_int32()
        st = lib().orc_bj_inv(self.h, _p(dinv), C.byref(bad))
        if st != OK:
            raise OracleError(st, f"bj_inv (block {bad.value})")
        return dinv

    def ssor_ai_apply(self, r, omega=1.0):
        dinv = self.bj_inv()
        r = np.ascontiguousarray(r, np.float64)
        z = np.empty_like(r)
        st = lib().orc_ssor_ai_apply(self.h, _p(dinv), float(omega), _p(r), _p(z))
        if st != OK:
            raise OracleError(st, "ssor_ai_apply")
        return z

    def ilu0_apply(self, r):
        st = lib().orc_ilu0_factor(self.h)
        if st != OK:
            raise OracleError(st, "ilu0_factor")
        r = np.ascontiguousarray(r, np.float64)
        z = np.empty_like(r)
        lib().orc_ilu0_apply(self.h, _p(r), _p(z))
        return z

    def pcg(self, F, d0=None, tol=1e-10, maxit=10000, precond="bj", omega=1.0, trace=False):
        """O-5 textbook PCG.  Returns (d, iters, rel_res, status[, trace[k, 6n]])."""
        N = 6 * self.n
        F = np.ascontiguousarray(F, np.float64)
        d0 = np.zeros(N) if d0 is None else np.ascontiguousarray(d0, np.float64)
        d = np.empty(N)
        it, rr = C.c_int32(), C.c_double()
        tr = np.zeros((maxit + 1, N)) if trace else None
        st = lib().orc_pcg(self.h, _p(F), _p(d0), _p(d), float(tol), int(maxit), PC[precond], float(omega),
                           C.byref(it), C.byref(rr), _p(tr) if trace else None)
        if st not in (OK, ERR_NO_CONVERGENCE, ERR_BREAKDOWN):
            raise OracleError(st, "pcg")
        out = (d, int(it.value), float(rr.value), int(st))
        if trace:
            out = out + (tr[: int(it.value) + 1],)
        return out

    def ldlt_solve(self, b):
        b = np.ascontiguousarray(b, np.float64)
        x = np.empty_like(b)
        st = lib().orc_ldlt_solve(self.h, _p(b), _p(x))
        if st != OK:
            raise OracleError(st, "ldlt_solve")
        return x


def assemble(P) -> OracleMatrix:
    return OracleMatrix.from_problem(P)


# ---------------------------------------------------------------- NEXT-3: contacts (O-8, O-9)

CONTACT_FIELDS = ("i", "v", "j", "e", "type", "t", "dist2")


def detect_contacts(vptr, vxy, d0, v_begin=0, v_end=None) -> dict:
    """O-8: every (vertex v of block i, edge e of block j != i) with distance < d0, in increasing
    (v, e); fields i, v, j, e (int32), type (0 VE, 1 VV), t (edge ratio), dist2."""
    vptr = np.ascontiguousarray(vptr, np.int32)
    vxy = np.ascontiguousarray(vxy, np.float64).reshape(-1, 2)
    n = vptr.shape[0] - 1
    v_end = int(vptr[-1]) if v_end is None else int(v_end)
    L = lib()
    out = None
    cap = 0
    while True:
        out = {k: np.empty(max(cap, 1), np.int32) for k in CONTACT_FIELDS[:5]}
        out["t"] = np.empty(max(cap, 1))
        out["dist2"] = np.empty(max(cap, 1))
        cnt = L.orc_detect_contacts(n, _p(vptr), _p(vxy), float(d0), int(v_begin), v_end, cap,
                                    *[_p(out[k]) for k in CONTACT_FIELDS])
        if cnt < 0:
            raise OracleError(ERR_ARG, "detect_contacts")
        if cnt <= cap:
            return {k: a[:cnt] for k, a in out.items()}
        cap = int(cnt)


def contact_springs(vptr, vxy, cxy, C_, p_n, shear_ratio) -> dict:
    """O-9: normal + shear spring of every VE contact, in record order (bi, bj, pen, e, g)."""
    vptr = np.ascontiguousarray(vptr, np.int32)
    vxy = np.ascontiguousarray(vxy, np.float64).reshape(-1, 2)
    cxy = np.ascontiguousarray(cxy, np.float64).reshape(-1, 2)
    nc = int(C_["i"].shape[0])
    nve = int((C_["type"] == 0).sum())
    m = 2 * nve
    o = {"bi": np.empty(max(m, 1), np.int32), "bj": np.empty(max(m, 1), np.int32), "pen": np.empty(max(m, 1)),
         "e": np.empty((max(m, 1), 6)), "g": np.empty((max(m, 1), 6))}
    f = [np.ascontiguousarray(C_[k], np.int32) for k in ("i", "v", "j", "e", "type")]
    t = np.ascontiguousarray(C_["t"], np.float64)
    got = lib().orc_contact_springs(vptr.shape[0] - 1, _p(vptr), _p(vxy), _p(cxy), nc, *[_p(a) for a in f], _p(t),
                                    float(p_n), float(shear_ratio), _p(o["bi"]), _p(o["bj"]), _p(o["pen"]),
                                    _p(o["e"]), _p(o["g"]))
    assert got == m
    return {k: a[:m] for k, a in o.items()}


CLASS_NAMES = {-1: "abandoned", 0: "VE", 1: "VV1", 2: "VV2"}


def classify_contacts(vptr, vxy, C_, sin_tol) -> np.ndarray:
    """O-10: the angle judgment and the VV1 / VV2 split of every record of O-8: class -1
    (abandoned), 0 (VE), 1 (VV1), 2 (VV2), per record."""
    vptr = np.ascontiguousarray(vptr, np.int32)
    vxy = np.ascontiguousarray(vxy, np.float64).reshape(-1, 2)
    nc = int(C_["i"].shape[0])
    cls = np.empty(max(nc, 1), np.int32)
    f = [np.ascontiguousarray(C_[k], np.int32) for k in ("i", "v", "j", "e", "type")]
    st = lib().orc_classify_contacts(vptr.shape[0] - 1, _p(vptr), _p(vxy), nc, *[_p(a) for a in f],
                                     float(sin_tol), _p(cls))
    if st != OK:
        raise OracleError(st, "classify_contacts")
    return cls[:nc]


def classified_contacts(vptr, vxy, C_, sin_tol) -> dict:
    """The classified contact set ("valid data will be stored in a successive array"): the
    records that pass the angle judgment, grouped by class (VE, VV1, VV2; stable, so increasing
    (v, e) within a class), with `type` = the class."""
    cls = classify_contacts(vptr, vxy, C_, sin_tol)
    keep = np.nonzero(cls >= 0)[0]
    order = keep[np.argsort(cls[keep], kind="stable")]
    out = {k: np.ascontiguousarray(C_[k][order]) for k in CONTACT_FIELDS}
    out["type"] = cls[order].astype(np.int32)
    return out


def classified_springs(vptr, vxy, cxy, Cc, p_n, shear_ratio) -> dict:
    """O-9 applied to EVERY record of a classified set (VE, VV1 and VV2 alike: normal + shear
    spring at the record's edge and edge ratio, t = 0 or 1 for the VV classes), in record order."""
    allve = dict(Cc)
    allve["type"] = np.zeros_like(Cc["type"])
    return contact_springs(vptr, vxy, cxy, allve, p_n, shear_ratio)


STATE_NAMES = {0: "open", 1: "slide", 2: "lock"}


def contact_check(vptr, vxy, Cc, d, e, g, p_n, shear_ratio, tan_phi, open_tol, state):
    """O-11: one interpenetration check / open-close switch over a classified set Cc whose springs
    (e, g: [2 count, 6], O-9 order) were formed for it.  Returns (new state, category 0..5 per
    contact, penalties [2 count] for the next assembly); `state` is not modified."""
    vptr = np.ascontiguousarray(vptr, np.int32)
    vxy = np.ascontiguousarray(vxy, np.float64).reshape(-1, 2)
    nc = int(Cc["i"].shape[0])
    st = np.array(state, np.int32, copy=True).reshape(-1)
    assert st.shape[0] == nc
    pen = np.empty(max(2 * nc, 1))
    cat = np.empty(max(nc, 1), np.int32)
    f = [np.ascontiguousarray(Cc[k], np.int32) for k in ("i", "v", "j", "e", "type")]
    dd = np.ascontiguousarray(d, np.float64)
    ee = np.ascontiguousarray(e, np.float64).reshape(-1, 6)
    gg = np.ascontiguousarray(g, np.float64).reshape(-1, 6)
    assert ee.shape[0] == 2 * nc and gg.shape[0] == 2 * nc
    r = lib().orc_contact_check(vptr.shape[0] - 1, _p(vptr), _p(vxy), nc, *[_p(a) for a in f], _p(dd), _p(ee),
                                _p(gg), float(p_n), float(shear_ratio), float(tan_phi), float(open_tol), _p(st), _p(pen),
                                _p(cat))
    if r != OK:
        raise OracleError(r, "contact_check")
    return st[:nc], cat[:nc], pen[:2 * nc]


def contact_loads(n, vptr, vxy, Cc, e, g, pen):
    """O-12: the gap load Fc [6n] of the closed normal springs (pen [2 count]) and the initial states
    (lock if the vertex touches or penetrates its edge, else open)."""
    vptr = np.ascontiguousarray(vptr, np.int32)
    vxy = np.ascontiguousarray(vxy, np.float64).reshape(-1, 2)
    nc = int(Cc["i"].shape[0])
    Fc = np.empty(6 * n)
    st0 = np.empty(max(nc, 1), np.int32)
    f = [np.ascontiguousarray(Cc[k], np.int32) for k in ("i", "v", "j", "e")]
    ee = np.ascontiguousarray(e, np.float64).reshape(-1, 6)
    gg = np.ascontiguousarray(g, np.float64).reshape(-1, 6)
    pp = np.ascontiguousarray(pen, np.float64) if pen is not None else None
    r = lib().orc_contact_loads(int(n), _p(vptr), _p(vxy), nc, *[_p(a) for a in f], _p(ee), _p(gg),
                                _p(pp) if pp is not None else None, _p(Fc), _p(st0))
    if r != OK:
        raise OracleError(r, "contact_loads")
    return Fc, st0[:nc]


def state_penalties(state, p_n, shear_ratio):
    """Spring penalties of contact states (reading N4): normal p_n if closed (slide / lock), shear
    shear_ratio * p_n if lock, else 0 (the spring stays in the list with p = 0, reading Z10)."""
    state = np.asarray(state)
    pen = np.zeros(2 * state.size)
    pen[0::2] = np.where(state >= 1, p_n, 0.0)
    pen[1::2] = np.where(state == 2, shear_ratio * p_n, 0.0)
    return pen


def open_close_loop(n, kdiag, F, vptr, vxy, cxy, Cc, p_n, shear_ratio, tan_phi, open_tol, tol=1e-10, max_oc=30,
                    precond="bj"):
    """Loop 3 on the oracle, reading N4: initial states from the gaps (O-12); then repeat
    { assemble K (O-1) with the penalties of the states; F_eff = F + gap load (O-12); solve (O-5)
    warm-started from the previous solution; check (O-11) } until no contact changes state
    (no C1, C2, C4, C5).  Returns (d, states, history [(pcg iters, category counts)], converged)."""
    sp = classified_springs(vptr, vxy, cxy, Cc, p_n, shear_ratio)
    _, state = contact_loads(n, vptr, vxy, Cc, sp["e"], sp["g"], None)
    pen = state_penalties(state, p_n, shear_ratio)
    d = np.zeros(6 * n)
    hist = []
    for _ in range(max_oc):
        Fc, _ = contact_loads(n, vptr, vxy, Cc, sp["e"], sp["g"], pen)
        M = OracleMatrix(n, kdiag, sp["bi"], sp["bj"], pen, sp["e"], sp["g"])
        d, it, rr, st = M.pcg(F + Fc, d0=d, tol=tol, precond=precond)
        if st != OK:
            raise OracleError(st, "open_close_loop pcg")
        state, cat, pen = contact_check(vptr, vxy, Cc, d, sp["e"], sp["g"], p_n, shear_ratio, tan_phi, open_tol,
                                        state)
        counts = np.bincount(cat, minlength=6)
        hist.append((it, counts))
        if counts[1] + counts[2] + counts[4] + counts[5] == 0:
            return d, state, hist, True
    return d, state, hist, False


def contact_transfer(prev, prev_state, cur, init_state):
    """O-13: the states of the current records, transferred from the previous step's record with the
    same (v, e), else the initial state.  Returns (state, matched)."""
    pv, pe = np.ascontiguousarray(prev["v"], np.int32), np.ascontiguousarray(prev["e"], np.int32)
    cv, ce = np.ascontiguousarray(cur["v"], np.int32), np.ascontiguousarray(cur["e"], np.int32)
    ps = np.ascontiguousarray(prev_state, np.int32)
    ini = np.ascontiguousarray(init_state, np.int32)
    out = np.empty(max(cv.size, 1), np.int32)
    matched = lib().orc_contact_transfer(pv.size, _p(pv), _p(pe), _p(ps), cv.size, _p(cv), _p(ce), _p(ini), _p(out))
    return out[:cv.size], int(matched)
