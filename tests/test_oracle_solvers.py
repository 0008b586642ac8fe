"""Pins for oracle O-4 (block inverse), O-5 (PCG), O-6 (SSOR-AI, ILU(0)), O-7 (LDL^T).

Each pin is something other than the oracle itself: numpy /
scipy library routines, closed-form special cases (block-diagonal K -> one
iteration; a chain of blocks -> ILU(0) exact; two blocks -> first-order SSOR
truncation exact; omega = 0 -> SSOR-AI == BJ), the CG optimality invariant
(energy-norm error non-increasing, reading Z18) and brute-force dense ILU(0).
"""
import numpy as np
import pytest
import scipy.linalg as sla
import scipy.sparse as sp
import scipy.sparse.linalg as spl

import oracle
from synth import make_slope, preset
from conftest import dense_from_springs


def _dense(M, n):
    ip, ix, dv = M.full_csr()
    return sp.csr_matrix((dv, ix, ip), shape=(6 * n, 6 * n)).toarray()


# ------------------------------------------------------------------ O-4 block inverse

def test_bj_inverse_vs_numpy(tiny, tiny_oracle):
    D = tiny_oracle.export().diag
    Dinv = tiny_oracle.bj_inv()
    ref = np.linalg.inv(D)
    kappa = np.linalg.cond(D)
    for i in range(tiny.n):
        res = np.linalg.norm(D[i] @ Dinv[i] - np.eye(6))
        assert res <= 1e-13 * kappa[i]
        assert np.allclose(Dinv[i], ref[i], rtol=1e-11 * kappa[i], atol=0)
    assert np.allclose(Dinv, np.transpose(Dinv, (0, 2, 1)), rtol=1e-12, atol=0)


def test_bj_inverse_not_spd():
    kd = np.tile(np.eye(6), (2, 1, 1)); kd[1, 3, 3] = -1.0
    M = oracle.OracleMatrix(2, kd, np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros(0),
                            np.zeros((0, 6)), np.zeros((0, 6)))
    with pytest.raises(oracle.OracleError) as ei:
        M.bj_inv()
    assert ei.value.code == oracle.ERR_NOT_SPD


# ------------------------------------------------------------------ O-7 dense LDL^T

def test_ldlt_vs_scipy_cholesky(tiny, tiny_oracle):
    K = dense_from_springs(tiny)
    ref = sla.cho_solve(sla.cho_factor(K), tiny.F)
    x = tiny_oracle.ldlt_solve(tiny.F)
    assert np.linalg.norm(x - ref) <= 1e-11 * np.linalg.norm(ref)


# ------------------------------------------------------------------ O-5 PCG

def test_pcg_bj_vs_direct_solution(tiny, tiny_oracle):
    K = dense_from_springs(tiny)
    ev = np.linalg.eigvalsh(K)
    kappa = ev.max() / ev.min()
    ref = sla.cho_solve(sla.cho_factor(K), tiny.F)
    d, it, rr, st = tiny_oracle.pcg(tiny.F, tol=1e-10)
    assert st == oracle.OK and rr <= 1e-10 * 1.05
    # true relative residual rr bounds the relative error by kappa * rr
    assert np.linalg.norm(d - ref) / np.linalg.norm(ref) <= kappa * max(rr, 1e-16)
    assert np.linalg.norm(d - tiny_oracle.ldlt_solve(tiny.F)) <= 1e-8 * np.linalg.norm(ref)


@pytest.mark.parametrize("pc", ["bj", "none"])
def test_pcg_iteration_count_vs_scipy_cg(tiny, tiny_oracle, pc):
    K = sp.csr_matrix(dense_from_springs(tiny))
    M = None
    if pc == "bj":
        Dinv = np.linalg.inv(np.array([K[6 * i:6 * i + 6, 6 * i:6 * i + 6].toarray() for i in range(tiny.n)]))
        M = spl.LinearOperator(K.shape, matvec=lambda v: np.einsum("bij,bj->bi", Dinv, v.reshape(-1, 6)).ravel())
    cnt = [0]
    spl.cg(K, tiny.F, rtol=1e-10, atol=0.0, maxiter=5000, M=M, callback=lambda x: cnt.__setitem__(0, cnt[0] + 1))
    _, it, rr, st = tiny_oracle.pcg(tiny.F, tol=1e-10, precond=pc)
    assert st == oracle.OK
    assert abs(it - cnt[0]) <= max(2, int(0.01 * cnt[0])), (it, cnt[0])


def test_pcg_block_diagonal_one_iteration():
    # no springs: K is block diagonal, BJ is the exact inverse -> exactly one iteration
    P = make_slope(preset("tiny"))
    M = oracle.OracleMatrix(P.n, P.kdiag, np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros(0),
                            np.zeros((0, 6)), np.zeros((0, 6)))
    d, it, rr, st = M.pcg(P.F, tol=1e-10)
    assert st == oracle.OK and it == 1 and rr <= 1e-10


def test_pcg_energy_norm_monotone(tiny, tiny_oracle):
    # F = K d_true; CG minimises ||d_true - d_k||_K over growing Krylov spaces (Z18)
    K = dense_from_springs(tiny)
    d_true = np.random.default_rng(4).standard_normal(6 * tiny.n) * 1e-3
    F = tiny_oracle.spmv(d_true)
    d, it, rr, st, tr = tiny_oracle.pcg(F, tol=1e-10, maxit=2000, trace=True)
    assert st == oracle.OK
    E = tr - d_true[None, :]
    en = np.sqrt(np.einsum("ki,ij,kj->k", E, K, E))
    assert (np.diff(en) <= 1e-12 * en[0]).all()
    assert en[-1] < 1e-6 * en[0]


def test_pcg_zero_rhs_and_warm_start(tiny, tiny_oracle):
    d, it, rr, st = tiny_oracle.pcg(np.zeros(6 * tiny.n), d0=np.ones(6 * tiny.n))
    assert st == oracle.OK and it == 0 and rr == 0.0 and not d.any()         # reading Z2
    d1, it1, _, _ = tiny_oracle.pcg(tiny.F, tol=1e-10)
    from synth import warm_start
    d2, it2, rr2, st2 = tiny_oracle.pcg(tiny.F, d0=warm_start(d1, 8), tol=1e-10)
    assert st2 == oracle.OK and rr2 <= 1.05e-10 and it2 < it1                  # warm start
    d3, it3, rr3, st3 = tiny_oracle.pcg(tiny.F, d0=d1, tol=1e-6)
    assert it3 == 0 and st3 == oracle.OK


def test_pcg_maxit_no_convergence(tiny_oracle, tiny):
    d, it, rr, st = tiny_oracle.pcg(tiny.F, tol=1e-10, maxit=5)
    assert st == oracle.ERR_NO_CONVERGENCE and it == 5 and rr > 1e-10


# ------------------------------------------------------------------ O-6 SSOR-AI

def _ssor_dense(K, n, omega):
    D = np.zeros_like(K); U = np.zeros_like(K)
    for i in range(n):
        D[6 * i:6 * i + 6, 6 * i:6 * i + 6] = K[6 * i:6 * i + 6, 6 * i:6 * i + 6]
        U[6 * i:6 * i + 6, 6 * i + 6:] = K[6 * i:6 * i + 6, 6 * i + 6:]
    return D, U


def test_ssor_ai_explicit_dense(tiny, tiny_oracle):
    K = _dense(tiny_oracle, tiny.n)
    D, U = _ssor_dense(K, tiny.n, 1.0)
    Di = np.linalg.inv(D)
    for w in (1.0, 0.7):
        A = np.eye(K.shape[0]) - w * Di @ U
        Minv = A @ Di @ A.T
        r = np.random.default_rng(2).standard_normal(K.shape[0])
        z = tiny_oracle.ssor_ai_apply(r, omega=w)
        assert np.linalg.norm(z - Minv @ r) <= 1e-11 * np.linalg.norm(Minv @ r)


def test_ssor_ai_two_blocks_is_exact_sgs():
    # two blocks: (D + wL)^{-1} has no second-order term, so the first-order
    # truncation equals the exact symmetric Gauss-Seidel inverse (D+wU)^{-1} D (D+wL)^{-1}
    rng = np.random.default_rng(6)
    kd = np.array([np.eye(6) * 5 + 0.1 * np.ones((6, 6)) for _ in range(2)])
    e = rng.standard_normal((3, 6)); g = rng.standard_normal((3, 6))
    M = oracle.OracleMatrix(2, kd, np.array([0, 1, 0], np.int32), np.array([1, 0, 1], np.int32),
                            np.array([1.0, 0.5, 2.0]), e, g)
    K = _dense(M, 2)
    D, U = _ssor_dense(K, 2, 1.0)
    L = U.T
    r = rng.standard_normal(12)
    for w in (1.0, 1.3):
        ref = np.linalg.solve(D + w * U, D @ np.linalg.solve(D + w * L, r))
        assert np.allclose(M.ssor_ai_apply(r, omega=w), ref, rtol=1e-12, atol=1e-14 * np.abs(ref).max())


def test_ssor_ai_omega_zero_equals_bj(tiny, tiny_oracle):
    a = tiny_oracle.pcg(tiny.F, precond="bj")
    b = tiny_oracle.pcg(tiny.F, precond="ssor_ai", omega=0.0)
    assert a[1] == b[1] and np.array_equal(a[0], b[0])


def test_ssor_ai_symmetric_positive(tiny, tiny_oracle):
    rng = np.random.default_rng(11)
    r1, r2 = rng.standard_normal((2, 6 * tiny.n))
    z1, z2 = tiny_oracle.ssor_ai_apply(r1), tiny_oracle.ssor_ai_apply(r2)
    assert abs(r2 @ z1 - r1 @ z2) <= 1e-12 * np.linalg.norm(r1) * np.linalg.norm(z2)
    assert r1 @ z1 > 0


# ------------------------------------------------------------------ O-6 ILU(0)

def test_ilu0_chain_is_exact():
    # a single course: tridiagonal block pattern -> no fill -> ILU(0) = LU (reading Z15)
    P = make_slope(preset("tiny", courses=1, base_bricks=12))
    M = oracle.assemble(P)
    K = _dense(M, P.n)
    r = np.random.default_rng(0).standard_normal(6 * P.n)
    z = M.ilu0_apply(r)
    assert np.linalg.norm(z - np.linalg.solve(K, r)) <= 1e-12 * np.linalg.norm(z)
    d, it, rr, st = M.pcg(P.F, precond="ilu0")
    assert st == oracle.OK and it == 1


def _dense_ilu0(K, n, pattern):
    """Brute-force scalar ILU(0) (IKJ) restricted to the dense-block pattern."""
    A = K.copy()
    N = K.shape[0]
    mask = np.kron(pattern, np.ones((6, 6), bool))
    for i in range(1, N):
        for k in range(i):
            if not mask[i, k]:
                continue
            A[i, k] /= A[k, k]
            js = np.nonzero(mask[i, k + 1:])[0] + k + 1
            A[i, js] -= A[i, k] * A[k, js]
    return np.tril(A, -1) + np.eye(N), np.triu(A)


def test_ilu0_vs_bruteforce_scalar(tiny):
    P = make_slope(preset("tiny", courses=4, base_bricks=5))
    M = oracle.assemble(P)
    K = _dense(M, P.n)
    S = M.export()
    pat = np.eye(P.n, dtype=bool)
    for i in range(P.n):
        for u in range(S.row_ptr[i], S.row_ptr[i + 1]):
            pat[i, S.col_idx[u]] = pat[S.col_idx[u], i] = True
    Lf, Uf = _dense_ilu0(K, P.n, pat)
    r = np.random.default_rng(3).standard_normal(6 * P.n)
    ref = sla.solve_triangular(Uf, sla.solve_triangular(Lf, r, lower=True, unit_diagonal=True))
    z = M.ilu0_apply(r)
    assert np.linalg.norm(z - ref) <= 1e-10 * np.linalg.norm(ref)
    # incomplete: not the exact inverse on a 2-D pattern with fill
    assert np.linalg.norm(z - np.linalg.solve(K, r)) > 1e-8 * np.linalg.norm(ref)


def test_preconditioner_ordering_matches_paper_trend(paper):
    # qualitative P:162 / Table I: iterations ILU < SSOR-AI < BJ
    M = oracle.assemble(paper)
    its = {pc: M.pcg(paper.F, tol=1e-10, precond=pc)[1] for pc in ("bj", "ssor_ai", "ilu0")}
    assert its["ilu0"] < its["ssor_ai"] < its["bj"]
    assert 200 <= its["bj"] <= 350          # calibrated to Table I's 275 BJ iterations
