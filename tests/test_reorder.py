"""NEXT-2: reverse Cuthill-McKee block order (dda_rcm_order, host code in
libdda; no GPU needed).  Pins: it is a permutation; on a shuffled slope it
restores a small bandwidth (max |i - j| over coupled blocks) close to the
course-major order's; the renumbered system is the same operator (oracle
eigenvalues / solution map back)."""
import numpy as np
import pytest

import oracle
from synth import make_slope, preset


@pytest.fixture(scope="module")
def dda():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


def bandwidth(bi, bj):
    return int(np.max(np.abs(np.asarray(bi, np.int64) - np.asarray(bj, np.int64))))


def test_rcm_is_permutation_and_reduces_bandwidth(dda):
    P0 = make_slope(preset(5000, seed=1050))
    P = make_slope(preset(5000, seed=1050, shuffle=True))
    perm = dda.rcm_order(P.n, P.bi, P.bj)
    assert np.array_equal(np.sort(perm), np.arange(P.n))
    kd, bi, bj, F = dda.renumber(perm, P.kdiag, P.bi, P.bj, P.F)
    b_shuf, b_rcm, b_course = bandwidth(P.bi, P.bj), bandwidth(bi, bj), bandwidth(P0.bi, P0.bj)
    assert b_rcm < b_shuf / 10
    assert b_rcm <= 2 * b_course


def test_rcm_same_solution(dda):
    P = make_slope(preset("tiny", shuffle=True))
    perm = dda.rcm_order(P.n, P.bi, P.bj)
    kd, bi, bj, F = dda.renumber(perm, P.kdiag, P.bi, P.bj, P.F)
    d0, _, _, _ = oracle.OracleMatrix(P.n, P.kdiag, P.bi, P.bj, P.pen, P.e, P.g).pcg(P.F, tol=1e-12)
    d1, _, _, _ = oracle.OracleMatrix(P.n, kd, bi, bj, P.pen, P.e, P.g).pcg(F, tol=1e-12)
    inv = np.argsort(perm)
    assert np.allclose(d1.reshape(-1, 6)[inv].ravel(), d0, rtol=1e-8, atol=1e-12 * np.abs(d0).max())


def test_rcm_disconnected_and_errors(dda):
    perm = dda.rcm_order(6, np.array([0, 2], np.int32), np.array([1, 3], np.int32))
    assert sorted(perm.tolist()) == list(range(6))
    with pytest.raises(dda.DDAError):
        dda.rcm_order(3, np.array([0], np.int32), np.array([0], np.int32))
