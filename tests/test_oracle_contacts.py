"""Pins for oracle O-8 (contact detection: distance judgment + VE/VV classification) and
O-9 (the springs of the VE contacts) — NEXT-3.

What fixes them:
* a hand-derived golden case with every number exact in binary (tests/golden/two_squares_contacts.json):
  two offset squares (two VE contacts and their four springs) and two aligned squares (eight VV);
* the slope generator's OWN contact list, built from the brick layout (which block edges are shared)
  and not from distances: every generator contact must be detected as VE with the generator's edge
  ratio, and the oracle's springs must equal the generator's independently coded e, g vectors;
* exact invariances: scaling the geometry and d0 by 2, relabelling the blocks; monotonicity in d0.
"""
import json
import os

import numpy as np
import pytest

import oracle
from synth import make_slope, preset
from synth.slope import _t_transpose_times

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "two_squares_contacts.json")


def _geom(P):
    vptr = (4 * np.arange(P.n + 1)).astype(np.int32)
    return vptr, P.verts.reshape(-1, 2), P.centroid


@pytest.mark.parametrize("case", ["offset", "aligned"])
def test_golden_two_squares(case):
    G = json.load(open(GOLDEN))
    c = G["cases"][case]
    vptr, vxy, cxy = np.array(c["vptr"], np.int32), np.array(c["vxy"], float), np.array(c["centroid"], float)
    got = oracle.detect_contacts(vptr, vxy, G["d0"])
    for k in oracle.CONTACT_FIELDS:
        assert np.array_equal(got[k], np.array(c["contacts"][k], got[k].dtype)), k
    sp = oracle.contact_springs(vptr, vxy, cxy, got, G["p_n"], G["shear_ratio"])
    for k in ("bi", "bj", "pen"):
        assert np.array_equal(sp[k], np.array(c["springs"][k], sp[k].dtype)), k
    for k in ("e", "g"):
        assert np.array_equal(sp[k], np.array(c["springs"][k], float).reshape(-1, 6)), k


def _keys(C):
    return C["v"].astype(np.int64) * (1 << 32) + C["e"].astype(np.int64)


@pytest.mark.parametrize("name", ["tiny", "tiny_shuffled"])
def test_detects_every_generator_contact(name):
    P = make_slope(preset("tiny", shuffle=(name == "tiny_shuffled")))
    vptr, vxy, cxy = _geom(P)
    C = oracle.detect_contacts(vptr, vxy, 0.35)
    G = P.contacts
    k_det = _keys(C)
    assert np.all(np.diff(k_det) > 0)                      # increasing (v, e): canonical order
    pos = np.searchsorted(k_det, _keys(G))
    assert (pos < k_det.size).all() and np.array_equal(k_det[pos], _keys(G))
    assert np.array_equal(C["i"][pos], G["i"]) and np.array_equal(C["j"][pos], G["j"])
    # the generator places its contacts at the ends of shared edges and clips the edge ratio to
    # [0, 1]; after the vertex jitter a projection can fall just outside the edge (then the record
    # is VV with t at the clipped end) — the edge ratio matches either way
    assert np.abs(C["t"][pos] - G["tau"]).max() <= 1e-12
    assert (C["type"][pos] == 0).mean() > 0.3
    # springs: the generator's own e, g (synth/slope.py, coded independently) for the same contacts
    # (springs are formed for VE records; the generator's contacts are all springs, so take them as VE)
    sub = {k: C[k][pos] for k in oracle.CONTACT_FIELDS}
    sub["type"] = np.zeros_like(sub["type"])
    sp = oracle.contact_springs(vptr, vxy, cxy, sub, 1.0, 0.4)
    V = P.verts.reshape(-1, 2)
    P1, Q1 = V[G["v"]], V[G["e"]]
    Q2 = V[4 * G["j"] + (G["e"] - 4 * G["j"] + 1) % 4]
    d = Q2 - Q1
    u = d / np.linalg.norm(d, axis=1)[:, None]
    nrm = np.stack([u[:, 1], -u[:, 0]], axis=1)
    ci, cj, tau = G["i"], G["j"], G["tau"]
    for s, vec in ((0, nrm), (1, u)):
        e_ref = _t_transpose_times(P1[:, 0] - P.centroid[ci, 0], P1[:, 1] - P.centroid[ci, 1], vec[:, 0], vec[:, 1])
        g1 = _t_transpose_times(Q1[:, 0] - P.centroid[cj, 0], Q1[:, 1] - P.centroid[cj, 1], vec[:, 0], vec[:, 1])
        g2 = _t_transpose_times(Q2[:, 0] - P.centroid[cj, 0], Q2[:, 1] - P.centroid[cj, 1], vec[:, 0], vec[:, 1])
        g_ref = -((1.0 - tau)[:, None] * g1 + tau[:, None] * g2)
        assert np.abs(sp["e"][s::2] - e_ref).max() <= 1e-12
        assert np.abs(sp["g"][s::2] - g_ref).max() <= 1e-12
    assert np.array_equal(sp["bi"][0::2], ci) and np.array_equal(sp["bj"][0::2], cj)


def test_invariances():
    P = make_slope(preset(300, seed=1041))
    vptr, vxy, _ = _geom(P)
    C = oracle.detect_contacts(vptr, vxy, 0.2)
    # scaling by 2 is exact in binary: same records, same t and type, dist2 x 4 exactly
    C2 = oracle.detect_contacts(vptr, 2.0 * vxy, 0.4)
    for k in ("i", "v", "j", "e", "type", "t"):
        assert np.array_equal(C[k], C2[k]), k
    assert np.array_equal(4.0 * C["dist2"], C2["dist2"])
    # relabelling the blocks permutes the records, nothing else
    rng = np.random.default_rng(5)
    perm = rng.permutation(P.n)                    # old block b -> new block perm[b]
    inv = np.argsort(perm)
    V3 = P.verts[inv].reshape(-1, 2)
    C3 = oracle.detect_contacts(vptr, V3, 0.2)
    vmap = (4 * perm[C["i"]] + (C["v"] - 4 * C["i"])).astype(np.int64)
    emap = (4 * perm[C["j"]] + (C["e"] - 4 * C["j"])).astype(np.int64)
    order = np.argsort(vmap * (1 << 32) + emap)
    assert np.array_equal(C3["v"], vmap[order]) and np.array_equal(C3["e"], emap[order])
    assert np.array_equal(C3["t"], C["t"][order]) and np.array_equal(C3["dist2"], C["dist2"][order])
    # monotone in d0: a larger threshold keeps every record
    C4 = oracle.detect_contacts(vptr, vxy, 0.3)
    assert np.isin(_keys(C), _keys(C4)).all() and C4["v"].size >= C["v"].size
    C6 = oracle.detect_contacts(vptr, vxy, 0.02)
    assert np.isin(_keys(C6), _keys(C)).all() and C6["v"].size < C["v"].size
    # a vertex-range call is the corresponding slice of the full call
    a, b = 37, 180
    C5 = oracle.detect_contacts(vptr, vxy, 0.2, a, b)
    sel = (C["v"] >= a) & (C["v"] < b)
    assert np.array_equal(C5["e"], C["e"][sel]) and np.array_equal(C5["dist2"], C["dist2"][sel])


# ------------------------------------------------------------------ O-10: angle judgment, VV1 / VV2

ANGLE = os.path.join(os.path.dirname(__file__), "golden", "contact_angle_classes.json")


@pytest.mark.parametrize("case", ["aligned", "corner", "dart"])
def test_golden_angle_classes(case):
    G = json.load(open(ANGLE))
    c = G["cases"][case]
    vptr, vxy = np.array(c["vptr"], np.int32), np.array(c["vxy"], float)
    C = oracle.detect_contacts(vptr, vxy, G["d0"])
    assert np.array_equal(C["v"], c["v"]) and np.array_equal(C["e"], c["e"])
    for tol, want in c["classes"].items():
        assert np.array_equal(oracle.classify_contacts(vptr, vxy, C, float(tol)), want), tol
    if "first_springs" in c:
        Cc = oracle.classified_contacts(vptr, vxy, C, 0.35)
        sp = oracle.classified_springs(vptr, vxy, np.array(c["centroid"], float), Cc, 3.0, 0.5)
        assert np.array_equal(sp["e"][:2], np.array(c["first_springs"]["e"], float))
        assert np.array_equal(sp["g"][:2], np.array(c["first_springs"]["g"], float))
        assert np.array_equal(sp["pen"][:2], [3.0, 1.5])


def _rot90(vxy):
    """(x, y) -> (-y, x): exact in binary, preserves orientation, lengths and angles."""
    return np.stack([-vxy[:, 1], vxy[:, 0]], axis=1)


@pytest.mark.parametrize("name", ["tiny", "ragged"])
def test_angle_classes_invariant_and_generator_contacts(name):
    """Exact invariances of O-10 (rotation by 90 degrees, scaling by 2); every contact of the slope
    generator's own layout list (shared brick edges) passes the angle judgment, as VE or, at an
    edge end, VV1; the classified set is the passing records grouped VE, VV1, VV2."""
    P = make_slope(preset("tiny") if name == "tiny" else preset(400, seed=1047))
    vptr, vxy, cxy = _geom(P)
    C = oracle.detect_contacts(vptr, vxy, 0.35)
    cls = oracle.classify_contacts(vptr, vxy, C, 0.35)
    assert set(np.unique(cls)) <= {-1, 0, 1, 2}
    assert ((cls == 0) <= (C["type"] == 0)).all() and ((cls >= 1) <= (C["type"] == 1)).all()
    Cr = oracle.detect_contacts(vptr, _rot90(vxy), 0.35)
    assert np.array_equal(Cr["v"], C["v"]) and np.array_equal(Cr["e"], C["e"])
    assert np.array_equal(oracle.classify_contacts(vptr, _rot90(vxy), Cr, 0.35), cls)
    C2 = oracle.detect_contacts(vptr, 2.0 * vxy, 0.7)
    assert np.array_equal(oracle.classify_contacts(vptr, 2.0 * vxy, C2, 0.35), cls)
    # the generator's layout contacts (ends of shared, hence antiparallel, brick edges): all kept, the
    # interior ones VE and those at an edge end VV1 (parallel edges)
    pos = np.searchsorted(_keys(C), _keys(P.contacts))
    assert np.array_equal(cls[pos], C["type"][pos])
    # monotone in the tolerance: a larger angle tolerance abandons no more records
    cls_big = oracle.classify_contacts(vptr, vxy, C, 0.6)
    assert ((cls >= 0) <= (cls_big >= 0)).all()
    Cc = oracle.classified_contacts(vptr, vxy, C, 0.35)
    assert np.array_equal(np.sort(Cc["type"], kind="stable"), Cc["type"])
    assert Cc["type"].size == (cls >= 0).sum()


def test_angle_classes_brute_force_angles():
    """Cross-check O-10 against a differently computed statement of the same rule (angles by
    arctan2, not squared products): the decisions agree wherever the margin exceeds 1e-9 rad."""
    P = make_slope(preset(400, seed=1047))
    vptr, vxy, _ = _geom(P)
    C = oracle.detect_contacts(vptr, vxy, 0.35)
    cls = oracle.classify_contacts(vptr, vxy, C, 0.35)
    th = np.arcsin(0.35)
    agree = 0
    for k in range(C["i"].size):
        i, v, j, e = (int(C[f][k]) for f in ("i", "v", "j", "e"))
        a0, a1 = vptr[i], vptr[i + 1]
        P0 = vxy[v]
        A = vxy[v - 1 if v > a0 else a1 - 1] - P0
        B = vxy[v + 1 if v + 1 < a1 else a0] - P0
        q2 = e + 1 if e + 1 < vptr[j + 1] else vptr[j]
        d = vxy[q2] - vxy[e]
        nrm = np.arctan2(-d[0], d[1])                         # direction of the outward normal
        def elev(x):                                          # angle of x above the edge line (toward N)
            ang = np.arctan2(x[1], x[0]) - nrm
            return np.pi / 2 - abs((ang + np.pi) % (2 * np.pi) - np.pi)
        def par(x):                                           # angle between x and the edge line
            ang = abs((np.arctan2(x[1], x[0]) - np.arctan2(d[1], d[0])) % np.pi)
            return min(ang, np.pi - ang)
        turn = np.arctan2(A[0] * B[1] - A[1] * B[0], A @ B)
        margins = [abs(elev(A) + th), abs(elev(B) + th), abs(turn)]
        if min(margins) < 1e-9:
            continue
        ok = turn < 0 and elev(A) >= -th and elev(B) >= -th
        want = -1 if not ok else (0 if C["type"][k] == 0 else None)
        if want is None:
            pm = [abs(par(A) - th), abs(par(B) - th)]
            if min(pm) < 1e-9:
                continue
            want = 1 if (par(A) <= th or par(B) <= th) else 2
        assert cls[k] == want, (k, cls[k], want)
        agree += 1
    assert agree > 0.99 * C["i"].size
