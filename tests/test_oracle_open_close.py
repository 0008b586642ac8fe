"""Pins for oracle O-11 (interpenetration check / open-close switch: p1, p2 -> C1..C5, P:74,
P:112) and O-12 (contact initialisation and the gap load), and the oracle open-close loop (loop 3,
P:27) built from O-1, O-5, O-9, O-11, O-12 — NEXT-4.

What fixes them:
* a hand-derived golden (tests/golden/contact_states.json), every number exact in binary: the
  initial states, the gap load, and seven checks covering C1..C5, the open tolerance and "no switch";
* d = 0 changes no state (the initial states are a fixed point of the check at zero displacement);
* the loop's fixed point is an equilibrium of the contact energy: with the final states, the
  gradient of  1/2 d^T K0 d - F^T d + sum_closed 1/2 p_n (dn0 + un)^2 + sum_lock 1/2 p_s us^2
  (K0 = the diagonal terms; every spring term written out densely with numpy, independently of
  O-1 / O-12) vanishes, and every state is consistent with its own displacement.
"""
import json
import os

import numpy as np
import pytest

import oracle
from synth import make_slope, preset

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "contact_states.json")


def _setup(G, case):
    c = G[case]
    vptr, vxy, cxy = np.array(c["vptr"], np.int32), np.array(c["vxy"], float), np.array(c["centroid"], float)
    C = oracle.detect_contacts(vptr, vxy, G["d0"])
    Cc = oracle.classified_contacts(vptr, vxy, C, G["sin_tol"])
    sp = oracle.classified_springs(vptr, vxy, cxy, Cc, G["p_n"], G["shear_ratio"])
    return vptr, vxy, cxy, Cc, sp


@pytest.mark.parametrize("case", ["offset", "corner"])
def test_golden_checks(case):
    G = json.load(open(GOLDEN))
    vptr, vxy, cxy, Cc, sp = _setup(G, case)
    assert Cc["i"].size == 2 and (Cc["type"] == (0 if case == "offset" else 2)).all()
    for name, ck in G[case]["checks"].items():
        d = np.zeros(12)
        d[6:8] = ck["dB"]
        st, cat, pen = oracle.contact_check(vptr, vxy, Cc, d, sp["e"], sp["g"], G["p_n"], G["shear_ratio"],
                                            G["tan_phi"], G["open_tol"], np.array(ck["old"]))
        assert np.array_equal(st, ck["state"]), name
        assert np.array_equal(cat, ck["cat"]), name
        assert np.array_equal(pen, ck["pen"]), name


def test_golden_initial_states_and_gap_load():
    G = json.load(open(GOLDEN))
    vptr, vxy, cxy, Cc, sp = _setup(G, "offset")
    Fc, st0 = oracle.contact_loads(2, vptr, vxy, Cc, sp["e"], sp["g"], None)
    assert np.array_equal(st0, G["offset"]["state0"]) and not Fc.any()
    pen = oracle.state_penalties(np.array([2, 2]), G["p_n"], G["shear_ratio"])
    Fc, _ = oracle.contact_loads(2, vptr, vxy, Cc, sp["e"], sp["g"], pen)
    assert np.array_equal(Fc, G["offset"]["Fc_closed"])
    pen = oracle.state_penalties(np.array([0, 1]), G["p_n"], G["shear_ratio"])   # only contact 1 closed
    Fc, _ = oracle.contact_loads(2, vptr, vxy, Cc, sp["e"], sp["g"], pen)
    f = -3.0 / 64
    assert np.array_equal(Fc[:6], f * sp["g"][2]) and np.array_equal(Fc[6:], f * sp["e"][2])


def _slope_case(n=None, seed=1041):
    P = make_slope(preset("tiny") if n is None else preset(n, seed=seed))
    vptr = (4 * np.arange(P.n + 1)).astype(np.int32)
    vxy = P.verts.reshape(-1, 2)
    V = P.verts
    area = 0.5 * np.abs(np.sum(V[:, :, 0] * np.roll(V[:, :, 1], -1, 1) - np.roll(V[:, :, 0], -1, 1) * V[:, :, 1], 1))
    F = np.zeros((P.n, 6))
    F[:, 1] = -area                                            # self-weight on v0
    C = oracle.detect_contacts(vptr, vxy, 0.35)
    Cc = oracle.classified_contacts(vptr, vxy, C, 0.35)
    return P, vptr, vxy, F.reshape(-1), Cc


def test_zero_displacement_is_a_fixed_point():
    P, vptr, vxy, F, Cc = _slope_case()
    sp = oracle.classified_springs(vptr, vxy, P.centroid, Cc, 40.0, 0.4)
    _, st0 = oracle.contact_loads(P.n, vptr, vxy, Cc, sp["e"], sp["g"], None)
    assert 0 < (st0 == 2).sum() < st0.size
    st, cat, pen = oracle.contact_check(vptr, vxy, Cc, np.zeros(6 * P.n), sp["e"], sp["g"], 40.0, 0.4, 0.577, 0.01,
                                        st0)
    assert np.array_equal(st, st0)
    assert set(np.unique(cat)) <= {0, 3} and ((cat == 3) == (st0 == 2)).all()
    assert np.array_equal(pen, oracle.state_penalties(st0, 40.0, 0.4))


def test_open_close_loop_fixed_point_is_equilibrium():
    P, vptr, vxy, F, Cc = _slope_case()
    p_n, sr, tphi, otol = 40.0, 0.4, 0.577, 0.01
    d, st, hist, conv = oracle.open_close_loop(P.n, P.kdiag, F, vptr, vxy, P.centroid, Cc, p_n, sr, tphi, otol)
    assert conv and 2 <= len(hist) <= 30
    assert hist[0][1][1] > 0                                   # states did switch on the way (C1)
    sp = oracle.classified_springs(vptr, vxy, P.centroid, Cc, p_n, sr)
    # independent dense statement of the contact energy's gradient at d
    n, nc = P.n, Cc["i"].size
    K0 = np.zeros((6 * n, 6 * n))
    for b in range(n):
        U = np.triu(P.kdiag[b])
        K0[6 * b:6 * b + 6, 6 * b:6 * b + 6] = U + np.triu(U, 1).T
    grad = K0 @ d - F
    for k in range(nc):
        i, j = int(Cc["i"][k]), int(Cc["j"][k])
        a_n = np.zeros(6 * n); a_n[6 * i:6 * i + 6] = sp["e"][2 * k]; a_n[6 * j:6 * j + 6] += sp["g"][2 * k]
        a_s = np.zeros(6 * n); a_s[6 * i:6 * i + 6] = sp["e"][2 * k + 1]; a_s[6 * j:6 * j + 6] += sp["g"][2 * k + 1]
        q, v = int(Cc["e"][k]), int(Cc["v"][k])
        q2 = q + 1 if q + 1 < vptr[j + 1] else vptr[j]
        u = (vxy[q2] - vxy[q]) / np.linalg.norm(vxy[q2] - vxy[q])
        dn0 = np.array([u[1], -u[0]]) @ (vxy[v] - vxy[q])
        dn = dn0 + a_n @ d
        if st[k] >= 1:
            grad += p_n * dn * a_n
            assert dn <= otol + 1e-12                          # closed contacts are (nearly) in contact
        else:
            assert dn > -1e-12                                 # open contacts do not penetrate
        if st[k] == 2:
            grad += sr * p_n * (a_s @ d) * a_s
    assert np.linalg.norm(grad) <= 1e-8 * np.linalg.norm(F)


def test_open_close_loop_1k_converges():
    P, vptr, vxy, F, Cc = _slope_case(1000)
    d, st, hist, conv = oracle.open_close_loop(P.n, P.kdiag, F, vptr, vxy, P.centroid, Cc, 40.0, 0.4, 0.577, 0.01)
    assert conv and len(hist) <= 15
    assert (st == 0).any() and (st == 1).any() and (st == 2).any()


# ------------------------------------------------------------------ O-13: contact transfer

def _perturbed(P, scale, seed):
    """The slope's polygons moved by a small random displacement (the next step's geometry)."""
    rng = np.random.default_rng(seed)
    return P.verts.reshape(-1, 2) + rng.uniform(-scale, scale, (P.n * 4, 2))


def test_contact_transfer_against_brute_force():
    P, vptr, vxy, F, _ = _slope_case()
    # step 1: the contacts within 0.1 h, their converged open-close states
    Cc = oracle.classified_contacts(vptr, vxy, oracle.detect_contacts(vptr, vxy, 0.1), 0.35)
    d, st, hist, conv = oracle.open_close_loop(P.n, P.kdiag, F, vptr, vxy, P.centroid, Cc, 40.0, 0.4, 0.577, 0.01)
    assert conv
    # step 2: moved polygons, contacts within 0.35 h: most persist, some are new
    vxy2 = _perturbed(P, 0.05, 3)
    C2 = oracle.classified_contacts(vptr, vxy2, oracle.detect_contacts(vptr, vxy2, 0.35), 0.35)
    sp2 = oracle.classified_springs(vptr, vxy2, P.centroid, C2, 40.0, 0.4)
    _, init = oracle.contact_loads(P.n, vptr, vxy2, C2, sp2["e"], sp2["g"], None)
    got, matched = oracle.contact_transfer(Cc, st, C2, init)
    prev = {(int(v), int(e)): int(s) for v, e, s in zip(Cc["v"], Cc["e"], st)}
    want = np.array([prev.get((int(v), int(e)), int(s0)) for v, e, s0 in zip(C2["v"], C2["e"], init)])
    assert np.array_equal(got, want)
    assert matched == sum((int(v), int(e)) in prev for v, e in zip(C2["v"], C2["e"]))
    assert 0 < matched < C2["v"].size                      # some contacts persist, some are new
    # the identity step transfers everything; an empty previous step transfers nothing
    same, mt = oracle.contact_transfer(Cc, st, Cc, np.zeros_like(st))
    assert np.array_equal(same, st) and mt == st.size
    empty = {k: v[:0] for k, v in Cc.items()}
    none, m0 = oracle.contact_transfer(empty, st[:0], C2, init)
    assert np.array_equal(none, init) and m0 == 0
