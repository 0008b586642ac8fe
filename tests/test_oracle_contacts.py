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
