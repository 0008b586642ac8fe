"""Pins for oracle O-1 (assembly), O-2 (full expansion) and O-3 (SpMV).

What fixes each part:
* structure — brute force (set of unordered pairs) and scipy.sparse's own
  COO->CSR and CSR->CSC conversions (library), bit-exact;
* values — an independent dense numpy assembly from the springs and a
  hand-derived two-block golden case (tests/golden/two_block.json);
* SpMV — unit-vector columns (exact), scipy.sparse products, symmetry.
"""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from synth import make_slope, preset
from conftest import dense_from_springs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "two_block.json")


def _golden():
    with open(GOLDEN) as f:
        return json.load(f)


def test_golden_two_block():
    G = _golden()
    M = oracle.OracleMatrix(G["n"], np.array(G["kdiag"], float), np.array(G["bi"], np.int32),
                            np.array(G["bj"], np.int32), np.array(G["pen"], float),
                            np.array(G["e"], float), np.array(G["g"], float))
    S = M.export()
    X = G["expect"]
    for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
        assert getattr(S, k).tolist() == X[k], k
    assert np.array_equal(S.upper, np.array(X["upper"], float))
    assert np.array_equal(S.diag, np.array(X["diag"], float))
    assert np.array_equal(M.spmv(np.array(X["x"], float)), np.array(X["y"], float))


def test_structure_bruteforce_and_scipy(tiny, tiny_oracle):
    P, S = tiny, tiny_oracle.export()
    a = np.minimum(P.bi, P.bj); b = np.maximum(P.bi, P.bj)
    pairs = sorted(set(zip(a.tolist(), b.tolist())))
    got = [(r, c) for r in range(P.n) for c in S.col_idx[S.row_ptr[r]:S.row_ptr[r + 1]].tolist()]
    assert got == pairs                                                   # brute force
    coo = sp.coo_matrix((np.ones(P.m), (a, b)), shape=(P.n, P.n)).tocsr()
    coo.sum_duplicates(); coo.sort_indices()
    assert np.array_equal(S.row_ptr, coo.indptr) and np.array_equal(S.col_idx, coo.indices)
    # CSR with data = position+1, converted to CSC by scipy: the lower-CSR of the
    # transpose map (row-low-i / row-low-p)
    up = sp.csr_matrix((np.arange(1, tiny_oracle.nnzb + 1, dtype=float), S.col_idx, S.row_ptr),
                       shape=(P.n, P.n)).tocsc()
    up.sort_indices()
    assert np.array_equal(S.low_ptr, up.indptr)
    assert np.array_equal(S.low_row, up.indices)
    assert np.array_equal(S.low_to_up, up.data.astype(np.int64) - 1)
    # every stored block is strictly upper (reading Z6)
    rows = np.repeat(np.arange(P.n), np.diff(S.row_ptr))
    assert (S.col_idx > rows).all()


def test_values_vs_dense_numpy(tiny, tiny_oracle):
    P, S = tiny, tiny_oracle.export()
    K = dense_from_springs(P)
    scale = np.abs(K).max()
    for i in range(P.n):
        assert np.allclose(S.diag[i], K[6 * i:6 * i + 6, 6 * i:6 * i + 6], rtol=0, atol=1e-14 * scale)
        for u in range(S.row_ptr[i], S.row_ptr[i + 1]):
            j = S.col_idx[u]
            assert np.allclose(S.upper[u], K[6 * i:6 * i + 6, 6 * j:6 * j + 6], rtol=0, atol=1e-14 * scale)
    ip, ix, dv = tiny_oracle.full_csr()
    A = sp.csr_matrix((dv, ix, ip), shape=K.shape).toarray()
    assert np.allclose(A, K, rtol=0, atol=1e-14 * scale)
    assert np.array_equal(A, A.T)                                         # exactly symmetric
    assert np.linalg.eigvalsh(A).min() > 0                                # SPD


def test_diag_bitwise_symmetric(tiny_oracle):
    D = tiny_oracle.export().diag
    assert np.array_equal(D, np.transpose(D, (0, 2, 1)))


def test_single_spring_values_exact():
    # one spring per pair: each stored entry is exactly one rounded product (p*e[r])*g[c]
    rng = np.random.default_rng(3)
    n = 3
    kd = np.tile(np.eye(6), (n, 1, 1))
    bi = np.array([2, 0], np.int32); bj = np.array([1, 2], np.int32)
    pen = rng.uniform(1, 2, 2); e = rng.standard_normal((2, 6)); g = rng.standard_normal((2, 6))
    S = oracle.OracleMatrix(n, kd, bi, bj, pen, e, g).export()
    assert S.row_ptr.tolist() == [0, 1, 2, 2] and S.col_idx.tolist() == [2, 2]
    # pair (0,2) from spring 1 (i=0<j=2): K_02 = p e g^T
    assert np.array_equal(S.upper[0], (pen[1] * e[1])[:, None] * g[1][None, :])
    # pair (1,2) from spring 0 (i=2>j=1): stored K_21^T, entry [r][c] = (p*e[c])*g[r]
    assert np.array_equal(S.upper[1], ((pen[0] * e[0])[None, :] * g[0][:, None]))


def test_zero_penalty_creates_structure():
    n = 2
    S = oracle.OracleMatrix(n, np.tile(np.eye(6), (n, 1, 1)), np.array([0], np.int32), np.array([1], np.int32),
                            np.array([0.0]), np.ones((1, 6)), np.ones((1, 6))).export()
    assert S.col_idx.tolist() == [1] and not S.upper.any()                # reading Z10


def test_no_springs_block_diagonal():
    n = 4
    kd = np.tile(2 * np.eye(6), (n, 1, 1))
    M = oracle.OracleMatrix(n, kd, np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros(0),
                            np.zeros((0, 6)), np.zeros((0, 6)))
    assert M.nnzb == 0
    x = np.arange(24.0)
    assert np.array_equal(M.spmv(x), 2 * x)


@pytest.mark.parametrize("bad", ["self", "range", "neg_pen"])
def test_invalid_springs_rejected(bad):
    bi = np.array([0], np.int32); bj = np.array([1], np.int32); pen = np.array([1.0])
    if bad == "self":
        bj[0] = 0
    elif bad == "range":
        bj[0] = 5
    else:
        pen[0] = -1.0
    with pytest.raises(oracle.OracleError) as ei:
        oracle.OracleMatrix(2, np.tile(np.eye(6), (2, 1, 1)), bi, bj, pen, np.ones((1, 6)), np.ones((1, 6)))
    assert ei.value.code == oracle.ERR_ARG


def test_spmv_unit_vectors_exact(tiny, tiny_oracle):
    # K e_k is column k: one nonzero product per row plus exact zeros (Z16 pin)
    ip, ix, dv = tiny_oracle.full_csr()
    A = sp.csr_matrix((dv, ix, ip), shape=(6 * tiny.n, 6 * tiny.n)).toarray()
    for k in [0, 5, 6, 37, 6 * tiny.n // 2 + 3, 6 * tiny.n - 1]:
        x = np.zeros(6 * tiny.n); x[k] = 1.0
        assert np.array_equal(tiny_oracle.spmv(x), A[:, k])


def test_spmv_vs_scipy_and_symmetry(tiny, tiny_oracle):
    K = sp.csr_matrix(dense_from_springs(tiny))
    rng = np.random.default_rng(9)
    x = rng.uniform(-1, 1, 6 * tiny.n); z = rng.uniform(-1, 1, 6 * tiny.n)
    y = tiny_oracle.spmv(x)
    ref = K @ x
    bound = abs(K) @ np.abs(x)
    assert (np.abs(y - ref) <= 1e-13 * bound).all()
    # symmetric-half product == full product invariant: z^T (K x) == x^T (K z)
    assert abs(z @ y - x @ tiny_oracle.spmv(z)) <= 1e-12 * (np.abs(z) @ bound)


def test_spmv_rows_matches_full(tiny_oracle):
    x = np.random.default_rng(1).uniform(-1, 1, 6 * tiny_oracle.n)
    y = tiny_oracle.spmv(x)
    rows = np.arange(0, 6 * tiny_oracle.n, 7)
    assert np.array_equal(tiny_oracle.spmv_rows(rows, x), y[rows])


def test_shuffled_ordering_same_operator():
    a = make_slope(preset("tiny")); b = make_slope(preset("tiny", shuffle=True))
    Ma, Mb = oracle.assemble(a), oracle.assemble(b)
    assert Ma.nnzb == Mb.nnzb
    ea = np.sort(np.linalg.eigvalsh(dense_from_springs(a)))
    ip, ix, dv = Mb.full_csr()
    pa = np.sort(np.linalg.eigvalsh(sp.csr_matrix((dv, ix, ip), shape=(6 * b.n,) * 2).toarray()))
    assert np.allclose(ea, pa, rtol=1e-11, atol=1e-11 * ea.max())


def test_spmv_par_equals_spmv():
    """The OpenMP timing variant of O-3 sums every row in the same order: bitwise equal."""
    P = make_slope(preset(2000, seed=1041))
    M = oracle.assemble(P)
    x = np.random.default_rng(3).uniform(-1, 1, 6 * P.n)
    y, th = M.spmv_par(x)
    assert th >= 1 and np.array_equal(y, M.spmv(x))
