"""B200-native DDA equation-solving hot path: thin Python binding of libdda.so.

Argument marshalling only — every step of the path (assembly, SpMV,
block-Jacobi setup, PCG, SSOR-AI) runs in the CUDA kernels behind the C ABI
declared in include/dda.h.  PyTorch supplies device memory and streams.
There is no CPU fallback: if the shared library is missing or no CUDA device
is present the calls raise.

Names follow the ABI: build_matrix, spmv, bj_setup, precond_apply, pcg_solve,
update_values, solve_host (§III.C P:100-110 and §IV).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libdda.so")

OK, ERR_ARG, ERR_CUDA, ERR_OOM, ERR_NOT_SPD, ERR_BREAKDOWN, ERR_NO_CONVERGENCE, ERR_NCCL = range(8)
PRECOND = {"none": 0, "bj": 1, "ssor_ai": 2, "ilu0": 3}

# symbols declared in include/dda.h (checked by tests/test_abi.py)
ABI_SYMBOLS = ("dda_build_matrix", "dda_update_values", "dda_matrix_info", "dda_matrix_export", "dda_spmv",
               "dda_bj_setup", "dda_precond_apply", "dda_pcg_solve", "dda_solve_host", "dda_launch_count",
               "dda_matrix_free", "dda_status_string", "dda_last_cuda_error", "dda_comm_unique_id",
               "dda_comm_init", "dda_comm_init_loopback", "dda_dist_attach", "dda_spmv_dist",
               "dda_pcg_solve_dist", "dda_comm_free", "dda_spmv_full", "dda_rcm_order",
               "dda_memory_release", "dda_memory_cached", "dda_detect_contacts", "dda_contacts_info",
               "dda_contacts_export", "dda_contact_springs", "dda_contacts_free", "dda_build_matrix_dist",
               "dda_dist_info", "dda_classify_contacts", "dda_contacts_classes",
               "dda_contact_init", "dda_contact_loads", "dda_contact_check", "dda_open_close",
               "dda_build_matrix_reordered", "dda_hsbcsr_build", "dda_hsbcsr_spmv", "dda_hsbcsr_export",
               "dda_hsbcsr_free", "dda_contact_transfer", "dda_solve_host_batch", "dda_pcg_set_history",
               "dda_comm_init_ipc", "dda_comm_ipc_export", "dda_comm_ipc_import")

_lib = None


class DDAError(RuntimeError):
    def __init__(self, status: int, what: str):
        name = lib().dda_status_string(status).decode() if _lib is not None else str(status)
        detail = lib().dda_last_cuda_error().decode() if (_lib is not None and status == ERR_CUDA) else ""
        super().__init__(f"{what}: {name}{' (' + detail + ')' if detail else ''}")
        self.status = status


def lib() -> C.CDLL:
    """Load libdda.so (build it first with __graft_entry__.build() or _build.py)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python __graft_entry__.py build` (no CPU fallback)")
        L = C.CDLL(LIB_PATH)
        P, I32, I64, D = C.c_void_p, C.c_int32, C.c_int64, C.c_double
        st = C.c_int
        L.dda_build_matrix.argtypes = [I32, P, I64, P, P, P, P, P, P, C.POINTER(P)]
        L.dda_build_matrix.restype = st
        L.dda_build_matrix_reordered.argtypes = [I32, P, I64, P, P, P, P, P, P, C.POINTER(P)]
        L.dda_build_matrix_reordered.restype = st
        L.dda_hsbcsr_build.argtypes = [P, P, C.POINTER(P)]
        L.dda_hsbcsr_build.restype = st
        L.dda_hsbcsr_spmv.argtypes = [P, P, P, P]
        L.dda_hsbcsr_spmv.restype = st
        L.dda_hsbcsr_export.argtypes = [P, P, P, P]
        L.dda_hsbcsr_export.restype = st
        L.dda_hsbcsr_free.argtypes = [P]
        L.dda_hsbcsr_free.restype = None
        L.dda_update_values.argtypes = [P, P, I64, P, P, P, P]
        L.dda_update_values.restype = st
        L.dda_matrix_info.argtypes = [P, C.POINTER(I32), C.POINTER(I64)]
        L.dda_matrix_info.restype = st
        L.dda_matrix_export.argtypes = [P] * 8
        L.dda_matrix_export.restype = st
        L.dda_spmv.argtypes = [P, P, P, P]
        L.dda_spmv.restype = st
        L.dda_spmv_full.argtypes = [P, P, P, P]
        L.dda_spmv_full.restype = st
        L.dda_bj_setup.argtypes = [P, P, C.POINTER(I32), P]
        L.dda_bj_setup.restype = st
        L.dda_precond_apply.argtypes = [P, st, D, P, P, P]
        L.dda_precond_apply.restype = st
        L.dda_pcg_solve.argtypes = [P, P, P, P, D, I32, st, D, C.POINTER(I32), C.POINTER(D), P]
        L.dda_pcg_solve.restype = st
        L.dda_solve_host.argtypes = [I32, P, I64, P, P, P, P, P, P, P, P, D, I32, st, D,
                                     C.POINTER(I32), C.POINTER(D), P]
        L.dda_solve_host.restype = st
        L.dda_solve_host_batch.argtypes = [I32, C.POINTER(HostSystem), D, I32, st, D, P]
        L.dda_solve_host_batch.restype = st
        L.dda_pcg_set_history.argtypes = [P, P, I32]
        L.dda_pcg_set_history.restype = st
        L.dda_launch_count.argtypes = []
        L.dda_launch_count.restype = I64
        L.dda_matrix_free.argtypes = [P]
        L.dda_matrix_free.restype = None
        L.dda_status_string.argtypes = [st]
        L.dda_status_string.restype = C.c_char_p
        L.dda_last_cuda_error.argtypes = []
        L.dda_last_cuda_error.restype = C.c_char_p
        L.dda_comm_unique_id.argtypes = [P]
        L.dda_comm_unique_id.restype = st
        L.dda_comm_init.argtypes = [I32, I32, P, C.POINTER(P)]
        L.dda_comm_init.restype = st
        L.dda_comm_init_loopback.argtypes = [I32, C.POINTER(P)]
        L.dda_comm_init_loopback.restype = st
        L.dda_comm_init_ipc.argtypes = [I32, I32, C.POINTER(P)]
        L.dda_comm_init_ipc.restype = st
        L.dda_comm_ipc_export.argtypes = [P, P, C.POINTER(I64)]
        L.dda_comm_ipc_export.restype = st
        L.dda_comm_ipc_import.argtypes = [P, P, I64]
        L.dda_comm_ipc_import.restype = st
        L.dda_dist_attach.argtypes = [P, I32, P, I32, P, P, P, P]
        L.dda_dist_attach.restype = st
        L.dda_spmv_dist.argtypes = [P, P, P, P]
        L.dda_spmv_dist.restype = st
        L.dda_pcg_solve_dist.argtypes = [P, P, P, P, D, I32, st, C.POINTER(I32), C.POINTER(D), P]
        L.dda_pcg_solve_dist.restype = st
        L.dda_comm_free.argtypes = [P]
        L.dda_comm_free.restype = None
        L.dda_rcm_order.argtypes = [I32, I64, P, P, P]
        L.dda_rcm_order.restype = st
        L.dda_memory_release.argtypes = []
        L.dda_memory_release.restype = None
        L.dda_memory_cached.argtypes = []
        L.dda_memory_cached.restype = I64
        L.dda_detect_contacts.argtypes = [I32, P, P, D, P, C.POINTER(P)]
        L.dda_detect_contacts.restype = st
        L.dda_contacts_info.argtypes = [P, C.POINTER(I64), C.POINTER(I64), C.POINTER(I64)]
        L.dda_contacts_info.restype = st
        L.dda_contacts_export.argtypes = [P] * 8
        L.dda_contacts_export.restype = st
        L.dda_contact_springs.argtypes = [P, P, D, D, P, P, P, P, P, P]
        L.dda_contact_springs.restype = st
        L.dda_contacts_free.argtypes = [P]
        L.dda_contacts_free.restype = None
        L.dda_build_matrix_dist.argtypes = [P, I32, I32, P, P, I64, P, P, P, P, P, P, C.POINTER(P)]
        L.dda_build_matrix_dist.restype = st
        L.dda_dist_info.argtypes = [P, I32, P, P, P, P, P]
        L.dda_dist_info.restype = st
        L.dda_classify_contacts.argtypes = [P, D, P]
        L.dda_classify_contacts.restype = st
        L.dda_contacts_classes.argtypes = [P, P, P, P, P]
        L.dda_contacts_classes.restype = st
        L.dda_contact_transfer.argtypes = [P, P, P, P, P, P]
        L.dda_contact_transfer.restype = st
        L.dda_contact_init.argtypes = [P, P, P]
        L.dda_contact_init.restype = st
        L.dda_contact_loads.argtypes = [P, P, P, P, P, P, P]
        L.dda_contact_loads.restype = st
        L.dda_contact_check.argtypes = [P, P, P, P, D, D, D, D, P, P, P, P, P, P]
        L.dda_contact_check.restype = st
        L.dda_open_close.argtypes = [P, P, P, P, P, P, D, D, D, D, D, I32, I32, P, P, P, P, P, P, P, P]
        L.dda_open_close.restype = st
        L.dda__last_checks.argtypes = [P]
        L.dda__last_checks.restype = C.c_int
        L.dda__pcg_engine.argtypes = [P, C.c_int]
        L.dda__pcg_engine.restype = C.c_int
        _lib = L
    return _lib


def _torch():
    import torch
    return torch


def _stream(stream=None) -> int:
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


def _dev(t, dtype, shape=None, name="tensor"):
    torch = _torch()
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} has shape {tuple(t.shape)}, expected {tuple(shape)}")
    return C.c_void_p(t.data_ptr())


def _check(st: int, what: str):
    if st != OK:
        raise DDAError(st, what)


def memory_release() -> None:
    """Return the library's cached device blocks to the driver (dda_memory_release)."""
    lib().dda_memory_release()


def memory_cached() -> int:
    """Bytes the library's caching allocator holds for reuse (dda_memory_cached)."""
    return int(lib().dda_memory_cached())


def launch_count() -> int:
    return int(lib().dda_launch_count())


class Matrix:
    """Upper-symmetric BSR6 stiffness matrix K owned by the library (A1)."""

    def __init__(self, handle: C.c_void_p):
        self._h = handle
        n, z = C.c_int32(), C.c_int64()
        _check(lib().dda_matrix_info(handle, C.byref(n), C.byref(z)), "dda_matrix_info")
        self.n, self.nnzb = int(n.value), int(z.value)

    @property
    def handle(self):
        if self._h is None:
            raise ValueError("matrix has been freed")
        return self._h

    def free(self):
        if self._h is not None and _lib is not None:
            _lib.dda_matrix_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def export(self) -> dict:
        n, z = self.n, self.nnzb
        out = {"row_ptr": np.empty(n + 1, np.int32), "col_idx": np.empty(z, np.int32),
               "low_ptr": np.empty(n + 1, np.int32), "low_row": np.empty(z, np.int32),
               "low_to_up": np.empty(z, np.int32), "diag": np.empty((n, 6, 6)), "upper": np.empty((z, 6, 6))}
        p = {k: v.ctypes.data_as(C.c_void_p) for k, v in out.items()}
        _check(lib().dda_matrix_export(self.handle, p["row_ptr"], p["col_idx"], p["low_ptr"], p["low_row"],
                                       p["low_to_up"], p["diag"], p["upper"]), "dda_matrix_export")
        return out

    def spmv(self, x, y=None, stream=None):
        torch = _torch()
        N = 6 * self.n
        xp = _dev(x, torch.float64, (N,), "x")
        if y is None:
            y = torch.empty_like(x)
        yp = _dev(y, torch.float64, (N,), "y")
        _check(lib().dda_spmv(self.handle, xp, yp, C.c_void_p(_stream(stream))), "dda_spmv")
        return y

    def spmv_full(self, x, y=None, stream=None):
        """configs[3] comparison: y = K x from full-storage BSR6 (expanded on first use)."""
        torch = _torch()
        N = 6 * self.n
        xp = _dev(x, torch.float64, (N,), "x")
        if y is None:
            y = torch.empty_like(x)
        yp = _dev(y, torch.float64, (N,), "y")
        _check(lib().dda_spmv_full(self.handle, xp, yp, C.c_void_p(_stream(stream))), "dda_spmv_full")
        return y

    def bj_setup(self, full: bool = False, stream=None):
        torch = _torch()
        out = torch.empty((self.n, 6, 6), dtype=torch.float64, device="cuda") if full else None
        bad = C.c_int32()
        st = lib().dda_bj_setup(self.handle, C.c_void_p(out.data_ptr()) if full else None, C.byref(bad),
                                C.c_void_p(_stream(stream)))
        if st != OK:
            raise DDAError(st, f"dda_bj_setup (block {bad.value})")
        return out

    def precond_apply(self, r, precond="bj", omega=1.0, stream=None):
        torch = _torch()
        N = 6 * self.n
        z = torch.empty_like(r)
        _check(lib().dda_precond_apply(self.handle, PRECOND[precond], float(omega),
                                       _dev(r, torch.float64, (N,), "r"), _dev(z, torch.float64, (N,), "z"),
                                       C.c_void_p(_stream(stream))), "dda_precond_apply")
        return z

    def pcg_solve(self, F, d0=None, d=None, tol=1e-10, maxit=10000, precond="bj", omega=1.0, stream=None,
                  raise_on_fail=False):
        """Returns (d, iters, rel_res, status); status OK / NO_CONVERGENCE / BREAKDOWN."""
        torch = _torch()
        N = 6 * self.n
        Fp = _dev(F, torch.float64, (N,), "F")
        d0p = _dev(d0, torch.float64, (N,), "d0") if d0 is not None else None
        if d is None:
            d = torch.empty_like(F)
        dp = _dev(d, torch.float64, (N,), "d")
        it, rr = C.c_int32(), C.c_double()
        st = lib().dda_pcg_solve(self.handle, Fp, d0p, dp, float(tol), int(maxit), PRECOND[precond], float(omega),
                                 C.byref(it), C.byref(rr), C.c_void_p(_stream(stream)))
        if st not in (OK, ERR_NO_CONVERGENCE, ERR_BREAKDOWN) or (raise_on_fail and st != OK):
            raise DDAError(st, "dda_pcg_solve")
        return d, int(it.value), float(rr.value), int(st)

    def set_history(self, hist=None):
        """dda_pcg_set_history: register a device float64 tensor of shape (cap, 2) that the following
        solves fill per iteration with (rho_k+1 = r^T M^-1 r, |r|^2 of the exact stopping test or NaN);
        None unregisters.  The tensor must stay alive while registered."""
        torch = _torch()
        if hist is None:
            _check(lib().dda_pcg_set_history(self.handle, None, 0), "dda_pcg_set_history")
            self._hist = None
            return
        if not (isinstance(hist, torch.Tensor) and hist.is_cuda and hist.dtype == torch.float64
                and hist.is_contiguous() and hist.dim() == 2 and hist.shape[1] == 2):
            raise ValueError("hist must be a contiguous CUDA float64 tensor of shape (cap, 2)")
        _check(lib().dda_pcg_set_history(self.handle, C.c_void_p(hist.data_ptr()), int(hist.shape[0])),
               "dda_pcg_set_history")
        self._hist = hist

    def pcg_engine(self, precond="bj") -> str:
        """The PCG engine dda_pcg_solve picks for this matrix (internal query, for byte accounting)."""
        return {0: "graph", 1: "persistent", 2: "scaled"}[lib().dda__pcg_engine(self.handle, PRECOND[precond])]

    def last_checks(self) -> int:
        """Exact stopping tests the last scaled-engine solve evaluated (internal query, byte accounting)."""
        return int(lib().dda__last_checks(self.handle))

    def update_values(self, kdiag, pen, e, g, stream=None):
        torch = _torch()
        m = int(pen.shape[0])
        _check(lib().dda_update_values(self.handle, _dev(kdiag, torch.float64, (self.n, 6, 6), "kdiag"), m,
                                       _dev(pen, torch.float64, (m,), "pen"), _dev(e, torch.float64, (m, 6), "e"),
                                       _dev(g, torch.float64, (m, 6), "g"), C.c_void_p(_stream(stream))),
               "dda_update_values")


class HSBCSR:
    """The paper's HSBCSR two-stage SpMV (dda_hsbcsr_*, NEXT-2 ablation) over a built Matrix."""

    def __init__(self, K: "Matrix", stream=None):
        self.K = K                       # the handle reads K's index arrays
        h = C.c_void_p()
        _check(lib().dda_hsbcsr_build(K.handle, C.c_void_p(_stream(stream)), C.byref(h)), "dda_hsbcsr_build")
        self._h = h

    def spmv(self, x, y=None, stream=None):
        torch = _torch()
        y = torch.empty_like(x) if y is None else y
        N = 6 * self.K.n
        _check(lib().dda_hsbcsr_spmv(self._h, _dev(x, torch.float64, (N,), "x"), _dev(y, torch.float64, (N,), "y"),
                                     C.c_void_p(_stream(stream))), "dda_hsbcsr_spmv")
        return y

    def export(self):
        """(d-data [6, dstride], nd-data-up [6, ustride]) host arrays."""
        strides = np.zeros(2, np.int64)
        _check(lib().dda_hsbcsr_export(self._h, None, None, strides.ctypes.data_as(C.c_void_p)), "dda_hsbcsr_export")
        dd = np.zeros((6, int(strides[0])))
        nd = np.zeros((6, max(int(strides[1]), 1)))
        _check(lib().dda_hsbcsr_export(self._h, dd.ctypes.data_as(C.c_void_p), nd.ctypes.data_as(C.c_void_p),
                                       strides.ctypes.data_as(C.c_void_p)), "dda_hsbcsr_export")
        return dd, nd[:, :int(strides[1])]

    def free(self):
        if self._h is not None and _lib is not None:
            _lib.dda_hsbcsr_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def build_matrix(kdiag, bi, bj, pen, e, g, stream=None, reorder=False) -> Matrix:
    """A1: assemble K from diagonal terms [n,6,6] and springs (bi, bj, pen, e[m,6], g[m,6]).
    reorder=True: dda_build_matrix_reordered (internal RCM order, caller's numbering at the ABI)."""
    torch = _torch()
    n = int(kdiag.shape[0])
    m = int(bi.shape[0])
    h = C.c_void_p()
    fn = lib().dda_build_matrix_reordered if reorder else lib().dda_build_matrix
    st = fn(n, _dev(kdiag, torch.float64, (n, 6, 6), "kdiag"), m,
                                _dev(bi, torch.int32, (m,), "bi"), _dev(bj, torch.int32, (m,), "bj"),
                                _dev(pen, torch.float64, (m,), "pen"), _dev(e, torch.float64, (m, 6), "e"),
                                _dev(g, torch.float64, (m, 6), "g"), C.c_void_p(_stream(stream)), C.byref(h))
    _check(st, "dda_build_matrix_reordered" if reorder else "dda_build_matrix")
    return Matrix(h)


def build_from_problem(P, device="cuda") -> Matrix:
    """Copy a synth.SlopeProblem to the device and assemble it."""
    t = problem_to_device(P, device)
    return build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])


def problem_to_device(P, device="cuda") -> dict:
    torch = _torch()
    return {"kdiag": torch.from_numpy(P.kdiag).to(device), "bi": torch.from_numpy(P.bi).to(device),
            "bj": torch.from_numpy(P.bj).to(device), "pen": torch.from_numpy(P.pen).to(device),
            "e": torch.from_numpy(P.e).to(device), "g": torch.from_numpy(P.g).to(device),
            "F": torch.from_numpy(P.F).to(device)}


class HostSystem(C.Structure):
    """dda_host_system (dda.h): one host system of dda_solve_host_batch."""
    _fields_ = [("n_blocks", C.c_int32), ("n_springs", C.c_int64), ("kdiag", C.c_void_p), ("bi", C.c_void_p),
                ("bj", C.c_void_p), ("pen", C.c_void_p), ("e", C.c_void_p), ("g", C.c_void_p), ("F", C.c_void_p),
                ("d0", C.c_void_p), ("d", C.c_void_p), ("iters", C.c_int32), ("rel_res", C.c_double),
                ("status", C.c_int)]


def _host_ptr(a, dtype):
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        import torch
        assert not a.is_cuda and a.is_contiguous() and a.dtype == {np.float64: torch.float64, np.int32: torch.int32}[dtype]
        return a.data_ptr()
    assert a.dtype == dtype and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def solve_host_batch(systems, tol=1e-10, maxit=10000, precond="bj", omega=1.0, stream=None):
    """Streamed end-to-end solves (dda_solve_host_batch): `systems` is a list of dicts with host arrays
    kdiag, bi, bj, pen, e, g, F, optional d0, and the output d (numpy or pinned CPU tensors, pinned for
    the copy overlap).  Returns [(iters, rel_res, status)] per system."""
    arr = (HostSystem * len(systems))()
    for k, S in enumerate(systems):
        h = arr[k]
        h.n_blocks = int(S["kdiag"].shape[0])
        h.n_springs = int(S["bi"].shape[0])
        for f, dt in (("kdiag", np.float64), ("bi", np.int32), ("bj", np.int32), ("pen", np.float64),
                      ("e", np.float64), ("g", np.float64), ("F", np.float64), ("d", np.float64)):
            setattr(h, f, _host_ptr(S[f], dt))
        h.d0 = _host_ptr(S.get("d0"), np.float64)
    st = lib().dda_solve_host_batch(len(systems), arr, float(tol), int(maxit), PRECOND[precond], float(omega),
                                    C.c_void_p(_stream(stream)))
    if st != OK:
        raise DDAError(st, "dda_solve_host_batch")
    return [(int(h.iters), float(h.rel_res), int(h.status)) for h in arr]


def solve_host(kdiag, bi, bj, pen, e, g, F, d0=None, tol=1e-10, maxit=10000, precond="bj", omega=1.0,
               out=None, stream=None):
    """End-to-end: host (numpy / pinned CPU tensor) inputs -> host solution, via dda_solve_host."""
    def ptr(a, dtype):
        if hasattr(a, "data_ptr"):
            return C.c_void_p(a.data_ptr())
        assert a.dtype == dtype and a.flags["C_CONTIGUOUS"]
        return a.ctypes.data_as(C.c_void_p)
    n = int(kdiag.shape[0]); m = int(bi.shape[0])
    if out is None:
        out = np.empty(6 * n)
    it, rr = C.c_int32(), C.c_double()
    st = lib().dda_solve_host(n, ptr(kdiag, np.float64), m, ptr(bi, np.int32), ptr(bj, np.int32),
                              ptr(pen, np.float64), ptr(e, np.float64), ptr(g, np.float64), ptr(F, np.float64),
                              ptr(d0, np.float64) if d0 is not None else None, ptr(out, np.float64), float(tol),
                              int(maxit), PRECOND[precond], float(omega), C.byref(it), C.byref(rr),
                              C.c_void_p(_stream(stream)))
    if st not in (OK, ERR_NO_CONVERGENCE, ERR_BREAKDOWN):
        raise DDAError(st, "dda_solve_host")
    return out, int(it.value), float(rr.value), int(st)


# ----------------------------------------------------------------------------- multi-GPU (§8(e))

class Comm:
    """Partitioned-solve communicator: NCCL (one partition per process / GPU) or
    loopback (all partitions in this process, for single-GPU testing)."""

    def __init__(self, handle, nparts_local: int):
        self._h = handle
        self.nparts_local = nparts_local
        self.parts = [None] * nparts_local     # (Matrix, LocalProblem) kept alive

    @staticmethod
    def unique_id() -> bytes:
        buf = C.create_string_buffer(128)
        _check(lib().dda_comm_unique_id(buf), "dda_comm_unique_id")
        return buf.raw

    @classmethod
    def nccl(cls, nranks: int, rank: int, uid: bytes) -> "Comm":
        h = C.c_void_p()
        buf = C.create_string_buffer(uid, 128)
        _check(lib().dda_comm_init(int(nranks), int(rank), buf, C.byref(h)), "dda_comm_init")
        return cls(h, 1)

    @classmethod
    def loopback(cls, nparts: int) -> "Comm":
        h = C.c_void_p()
        _check(lib().dda_comm_init_loopback(int(nparts), C.byref(h)), "dda_comm_init_loopback")
        return cls(h, nparts)

    @classmethod
    def ipc(cls, nranks: int, rank: int) -> "Comm":
        """dda_comm_init_ipc: one partition per process, peers' buffers mapped with CUDA IPC handles
        (exchange the ipc_export() blobs by any means, then ipc_import them in rank order)."""
        h = C.c_void_p()
        _check(lib().dda_comm_init_ipc(int(nranks), int(rank), C.byref(h)), "dda_comm_init_ipc")
        return cls(h, 1)

    def ipc_export(self) -> bytes:
        n = C.c_int64()
        _check(lib().dda_comm_ipc_export(self._h, None, C.byref(n)), "dda_comm_ipc_export")
        buf = C.create_string_buffer(n.value)
        _check(lib().dda_comm_ipc_export(self._h, buf, C.byref(n)), "dda_comm_ipc_export")
        return buf.raw[:n.value]

    def ipc_import(self, blobs):
        size = len(blobs[0])
        assert all(len(b) == size for b in blobs)
        buf = C.create_string_buffer(b"".join(blobs), size * len(blobs))
        _check(lib().dda_comm_ipc_import(self._h, buf, size), "dda_comm_ipc_import")

    def attach(self, part: int, K: "Matrix", lp, stream=None):
        sc = np.ascontiguousarray(lp.send_counts, np.int32)
        si = np.ascontiguousarray(lp.send_idx, np.int32)
        rc = np.ascontiguousarray(lp.recv_counts, np.int32)
        _check(lib().dda_dist_attach(self._h, int(part), K.handle, int(lp.n_own), sc.ctypes.data_as(C.c_void_p),
                                     si.ctypes.data_as(C.c_void_p), rc.ctypes.data_as(C.c_void_p),
                                     C.c_void_p(_stream(stream))), "dda_dist_attach")
        self.parts[part if self.nparts_local > 1 else 0] = (K, lp)

    def build_matrix_dist(self, part: int, n_global: int, bounds, kdiag_own, bi, bj, pen, e, g,
                          stream=None) -> "Matrix":
        """dda_build_matrix_dist: select this partition's springs (global ids, CUDA tensors), renumber,
        assemble and attach with the exchange plan, all in the library.  bounds: [nparts+1] row
        bounds (host); kdiag_own: [n_own, 6, 6] CUDA float64."""
        torch = _torch()
        m = int(bi.shape[0])
        b = np.ascontiguousarray(bounds, np.int32)
        me = part if (self.nparts_local > 1 and 0 <= part < b.shape[0] - 1) else None
        n_own = None if me is None else int(b[me + 1] - b[me])
        h = C.c_void_p()
        _check(lib().dda_build_matrix_dist(
            self._h, int(part), int(n_global), b.ctypes.data_as(C.c_void_p),
            _dev(kdiag_own, torch.float64, (n_own, 6, 6) if n_own is not None else None, "kdiag_own"), m,
            _dev(bi, torch.int32, (m,), "bi"), _dev(bj, torch.int32, (m,), "bj"),
            _dev(pen, torch.float64, (m,), "pen"), _dev(e, torch.float64, (m, 6), "e"),
            _dev(g, torch.float64, (m, 6), "g"), C.c_void_p(_stream(stream)), C.byref(h)), "dda_build_matrix_dist")
        K = Matrix(h)
        self.parts[part if self.nparts_local > 1 else 0] = (K, None)
        return K

    def info(self, part: int = 0, nparts: int = None) -> dict:
        """dda_dist_info: n_own, n_halo and the exchange plan of an attached partition."""
        P = nparts if nparts is not None else self.nparts_local
        n_own, n_halo = C.c_int32(), C.c_int32()
        sc, rc = np.zeros(P, np.int32), np.zeros(P, np.int32)
        _check(lib().dda_dist_info(self._h, int(part), C.cast(C.byref(n_own), C.c_void_p),
                                   C.cast(C.byref(n_halo), C.c_void_p), sc.ctypes.data_as(C.c_void_p),
                                   rc.ctypes.data_as(C.c_void_p), None), "dda_dist_info")
        si = np.zeros(max(int(sc.sum()), 1), np.int32)
        _check(lib().dda_dist_info(self._h, int(part), None, None, None, None, si.ctypes.data_as(C.c_void_p)),
               "dda_dist_info")
        return {"n_own": int(n_own.value), "n_halo": int(n_halo.value), "send_counts": sc, "recv_counts": rc,
                "send_idx": si[:int(sc.sum())]}

    @staticmethod
    def _ptrs(ts):
        arr = (C.c_void_p * len(ts))(*[C.c_void_p(t.data_ptr()) if t is not None else None for t in ts])
        return arr

    def spmv(self, xs, stream=None):
        torch = _torch()
        ys = [torch.empty_like(x) for x in xs]
        _check(lib().dda_spmv_dist(self._h, self._ptrs(xs), self._ptrs(ys), C.c_void_p(_stream(stream))),
               "dda_spmv_dist")
        return ys

    def pcg_solve(self, Fs, d0s=None, tol=1e-10, maxit=10000, precond="bj", stream=None):
        torch = _torch()
        ds = [torch.empty_like(F) for F in Fs]
        it, rr = C.c_int32(), C.c_double()
        st = lib().dda_pcg_solve_dist(self._h, self._ptrs(Fs), self._ptrs(d0s) if d0s is not None else None,
                                      self._ptrs(ds), float(tol), int(maxit), PRECOND[precond], C.byref(it),
                                      C.byref(rr), C.c_void_p(_stream(stream)))
        if st not in (OK, ERR_NO_CONVERGENCE, ERR_BREAKDOWN):
            raise DDAError(st, "dda_pcg_solve_dist")
        return ds, int(it.value), float(rr.value), int(st)

    def free(self):
        if self._h is not None and _lib is not None:
            _lib.dda_comm_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def row_bounds(n: int, nparts: int) -> np.ndarray:
    """Contiguous block-row ranges [b[p], b[p+1]) of equal size (int32, for dda_build_matrix_dist)."""
    if nparts < 1 or n < nparts:
        raise ValueError("need 1 <= nparts <= n")
    return np.array([(p * n) // nparts for p in range(nparts + 1)], dtype=np.int32)


def build_local(lp, device="cuda") -> Matrix:
    """Assemble a partition's local matrix (partition.LocalProblem) on the device."""
    torch = _torch()
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(device)
    return build_matrix(t(lp.kdiag), t(lp.bi), t(lp.bj), t(lp.pen), t(lp.e), t(lp.g))


# ----------------------------------------------------------------------------- NEXT-2 reordering

def rcm_order(n: int, bi, bj) -> np.ndarray:
    """Reverse Cuthill-McKee block order (perm[new] = old) of the contact graph, via dda_rcm_order."""
    bi = np.ascontiguousarray(bi, np.int32)
    bj = np.ascontiguousarray(bj, np.int32)
    perm = np.empty(int(n), np.int32)
    _check(lib().dda_rcm_order(int(n), int(bi.shape[0]), bi.ctypes.data_as(C.c_void_p),
                               bj.ctypes.data_as(C.c_void_p), perm.ctypes.data_as(C.c_void_p)), "dda_rcm_order")
    return perm


def renumber(perm, kdiag, bi, bj, F=None):
    """Apply a block order perm[new] = old to host inputs; returns (kdiag, bi, bj, F) in the new numbering.
    Map a solution back with d_old = d_new.reshape(-1, 6)[inv].ravel(), inv = argsort(perm)."""
    perm = np.asarray(perm)
    inv = np.empty_like(perm)
    inv[perm] = np.arange(perm.size, dtype=perm.dtype)
    out = (np.ascontiguousarray(np.asarray(kdiag)[perm]), inv[np.asarray(bi)].astype(np.int32),
           inv[np.asarray(bj)].astype(np.int32))
    if F is not None:
        out = out + (np.ascontiguousarray(np.asarray(F).reshape(-1, 6)[perm].reshape(-1)),)
    return out


# ---------------------------------------------------------------- NEXT-3: contact detection

class Contacts:
    """Library-owned contact records of dda_detect_contacts (include/dda.h)."""

    def __init__(self, handle, vptr, vxy):
        self._h = handle
        self._keep = (vptr, vxy)          # the library reads the geometry again in springs()
        cnt, nve, npr = C.c_int64(), C.c_int64(), C.c_int64()
        _check(lib().dda_contacts_info(self._h, C.byref(cnt), C.byref(nve), C.byref(npr)), "dda_contacts_info")
        self.count, self.n_ve, self.n_pairs = int(cnt.value), int(nve.value), int(npr.value)
        self.classified, self.n_vv1, self.n_vv2 = False, 0, 0

    def classify(self, sin_tol=0.35, stream=None):
        """dda_classify_contacts: angle judgment + VV1 / VV2 split; the set becomes the kept records
        grouped by class (type = 0 VE, 1 VV1, 2 VV2)."""
        _check(lib().dda_classify_contacts(self._h, C.c_double(sin_tol), C.c_void_p(_stream(stream))),
               "dda_classify_contacts")
        cnt, nve, npr = C.c_int64(), C.c_int64(), C.c_int64()
        _check(lib().dda_contacts_info(self._h, C.byref(cnt), C.byref(nve), C.byref(npr)), "dda_contacts_info")
        v1, v2, cl = C.c_int64(), C.c_int64(), C.c_int32()
        ref = lambda x: C.cast(C.byref(x), C.c_void_p)
        _check(lib().dda_contacts_classes(self._h, None, ref(v1), ref(v2), ref(cl)), "dda_contacts_classes")
        self.count, self.n_ve = int(cnt.value), int(nve.value)
        self.classified, self.n_vv1, self.n_vv2 = bool(cl.value), int(v1.value), int(v2.value)
        return self

    # ---- NEXT-4: interpenetration check / open-close switch (dda_contact_*)
    def init_states(self, stream=None):
        """dda_contact_init: gaps + endpoint sort; returns the initial states (CUDA int32 [count])."""
        torch = _torch()
        state = torch.empty(max(self.count, 1), dtype=torch.int32, device="cuda")
        _check(lib().dda_contact_init(self._h, C.c_void_p(state.data_ptr()), C.c_void_p(_stream(stream))),
               "dda_contact_init")
        return state[:self.count]

    def transfer_from(self, prev: "Contacts", prev_state, state, stream=None) -> int:
        """dda_contact_transfer: state (CUDA int32 [count], in: initial, out: transferred) of this set
        from the previous step's set and states; returns the number of transferred records."""
        mt = C.c_int64()
        _check(lib().dda_contact_transfer(prev._h, C.c_void_p(prev_state.data_ptr()), self._h,
                                          C.c_void_p(state.data_ptr()), C.cast(C.byref(mt), C.c_void_p),
                                          C.c_void_p(_stream(stream))), "dda_contact_transfer")
        return int(mt.value)

    def loads(self, sp, pen, F=None, stream=None):
        """dda_contact_loads: F (or 0) + the gap load of the closed normal springs (CUDA [6n])."""
        torch = _torch()
        n = self._keep[0].shape[0] - 1
        out = torch.empty(6 * n, dtype=torch.float64, device="cuda")
        _check(lib().dda_contact_loads(self._h, C.c_void_p(sp["e"].data_ptr()), C.c_void_p(sp["g"].data_ptr()),
                                       C.c_void_p(pen.data_ptr()), C.c_void_p(F.data_ptr()) if F is not None else None,
                                       C.c_void_p(out.data_ptr()), C.c_void_p(_stream(stream))), "dda_contact_loads")
        return out

    def check(self, d, sp, state, p_n=40.0, shear_ratio=0.4, tan_phi=0.577, open_tol=0.01, stream=None):
        """dda_contact_check: updates `state` in place; returns (pen, cat, cat_order, counts[6])."""
        torch = _torch()
        m = max(self.count, 1)
        pen = torch.empty(2 * m, dtype=torch.float64, device="cuda")
        cat = torch.empty(m, dtype=torch.int32, device="cuda")
        order = torch.empty(m, dtype=torch.int32, device="cuda")
        counts = np.zeros(6, np.int64)
        _check(lib().dda_contact_check(self._h, C.c_void_p(d.data_ptr()), C.c_void_p(sp["e"].data_ptr()),
                                       C.c_void_p(sp["g"].data_ptr()), float(p_n), float(shear_ratio), float(tan_phi),
                                       float(open_tol), C.c_void_p(state.data_ptr()), C.c_void_p(pen.data_ptr()),
                                       C.c_void_p(cat.data_ptr()), C.c_void_p(order.data_ptr()),
                                       counts.ctypes.data_as(C.c_void_p), C.c_void_p(_stream(stream))),
               "dda_contact_check")
        k = self.count
        return pen[:2 * k], cat[:k], order[:k], counts

    def open_close(self, K, kdiag, F, sp, state, d=None, p_n=40.0, shear_ratio=0.4, tan_phi=0.577, open_tol=0.01,
                   tol=1e-10, maxit=10000, max_oc=30, stream=None):
        """dda_open_close (loop 3): returns (d, state, pen, oc_iters, pcg_iters, converged, rel_res)."""
        torch = _torch()
        n = self._keep[0].shape[0] - 1
        d = torch.zeros(6 * n, dtype=torch.float64, device="cuda") if d is None else d
        pen = torch.empty(max(2 * self.count, 1), dtype=torch.float64, device="cuda")
        oc, pit, conv, rr = C.c_int32(), C.c_int32(), C.c_int32(), C.c_double()
        ref = lambda x: C.cast(C.byref(x), C.c_void_p)
        _check(lib().dda_open_close(K.handle, self._h, C.c_void_p(kdiag.data_ptr()), C.c_void_p(F.data_ptr()),
                                    C.c_void_p(sp["e"].data_ptr()), C.c_void_p(sp["g"].data_ptr()), float(p_n),
                                    float(shear_ratio), float(tan_phi), float(open_tol), float(tol), int(maxit),
                                    int(max_oc), C.c_void_p(state.data_ptr()), C.c_void_p(pen.data_ptr()),
                                    C.c_void_p(d.data_ptr()), ref(oc), ref(pit), ref(conv), ref(rr),
                                    C.c_void_p(_stream(stream))), "dda_open_close")
        return d, state, pen[:2 * self.count], int(oc.value), int(pit.value), bool(conv.value), float(rr.value)

    def free(self):
        if self._h is not None:
            lib().dda_contacts_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def export(self) -> dict:
        m = self.count
        o = {k: np.empty(m, np.int32) for k in ("i", "v", "j", "e", "type")}
        o["t"] = np.empty(m)
        o["dist2"] = np.empty(m)
        ptr = lambda a: a.ctypes.data_as(C.c_void_p)
        _check(lib().dda_contacts_export(self._h, *[ptr(o[k]) for k in ("i", "v", "j", "e", "type", "t", "dist2")]),
               "dda_contacts_export")
        return o

    def springs(self, cxy, p_n=40.0, shear_ratio=0.4, stream=None) -> dict:
        """Springs of the VE contacts as CUDA tensors (bi, bj, pen, e, g) for build_matrix."""
        torch = _torch()
        n = self._keep[0].shape[0] - 1
        m = 2 * (self.count if self.classified else self.n_ve)
        dev = self._keep[1].device
        o = {"bi": torch.empty(m, dtype=torch.int32, device=dev), "bj": torch.empty(m, dtype=torch.int32, device=dev),
             "pen": torch.empty(m, dtype=torch.float64, device=dev),
             "e": torch.empty((m, 6), dtype=torch.float64, device=dev),
             "g": torch.empty((m, 6), dtype=torch.float64, device=dev)}
        _check(lib().dda_contact_springs(self._h, _dev(cxy, torch.float64, (n, 2), "cxy"), float(p_n),
                                         float(shear_ratio), *[C.c_void_p(o[k].data_ptr()) for k in
                                                               ("bi", "bj", "pen", "e", "g")],
                                         C.c_void_p(_stream(stream))), "dda_contact_springs")
        return o


def detect_contacts(vptr, vxy, d0, stream=None) -> Contacts:
    """NEXT-3: dda_detect_contacts on CUDA tensors vptr [n+1] int32 and vxy [V, 2] float64."""
    torch = _torch()
    n = int(vptr.shape[0]) - 1
    vp = _dev(vptr, torch.int32, None, "vptr")
    vx = _dev(vxy, torch.float64, None, "vxy")
    h = C.c_void_p()
    _check(lib().dda_detect_contacts(n, vp, vx, float(d0), C.c_void_p(_stream(stream)), C.byref(h)),
           "dda_detect_contacts")
    return Contacts(h, vptr, vxy)
