"""NEXT-3 GPU parity: dda_detect_contacts / dda_contact_springs against the oracle's O-8 / O-9,
through the C ABI.  Integer fields and the decision bit-exact; t and dist2 bit-exact as well (both
sides round every product and sum as written); springs bit-exact.  Full size: sampled vertices."""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from synth import make_slope, preset

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "two_squares_contacts.json")
FIELDS = ("i", "v", "j", "e", "type", "t", "dist2")


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (no CPU fallback exists)")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


def _slope_geom(P):
    vptr = (4 * np.arange(P.n + 1)).astype(np.int32)
    return vptr, P.verts.reshape(-1, 2).copy(), P.centroid.copy()


def _random_polygons(n, seed):
    """Irregular convex polygons of 3-7 vertices on a jittered grid (ragged vertex counts)."""
    rng = np.random.default_rng(seed)
    side = int(np.ceil(np.sqrt(n)))
    k = rng.integers(3, 8, size=n)
    vptr = np.concatenate([[0], np.cumsum(k)]).astype(np.int32)
    pts, cen = [], []
    for b in range(n):
        c = np.array([b % side, b // side], float) * 1.0 + rng.uniform(-0.05, 0.05, 2)
        ang = np.sort(rng.uniform(0, 2 * np.pi, k[b]))
        r = rng.uniform(0.45, 0.6, k[b])
        pts.append(c + np.stack([r * np.cos(ang), r * np.sin(ang)], 1))
        cen.append(c)
    return vptr, np.concatenate(pts), np.array(cen)


def _gpu(dda, vptr, vxy, d0):
    Cg = dda.detect_contacts(torch.from_numpy(vptr).cuda(), torch.from_numpy(np.ascontiguousarray(vxy)).cuda(), d0)
    return Cg, Cg.export()


def _same(a, b):
    for k in FIELDS:
        assert a[k].shape == b[k].shape, (k, a[k].shape, b[k].shape)
        assert np.array_equal(a[k], b[k]), k


@pytest.mark.parametrize("case", ["offset", "aligned"])
def test_golden_two_squares(dda, case):
    G = json.load(open(GOLDEN))
    c = G["cases"][case]
    vptr, vxy = np.array(c["vptr"], np.int32), np.array(c["vxy"], float)
    Cg, got = _gpu(dda, vptr, vxy, G["d0"])
    for k in FIELDS:
        assert np.array_equal(got[k], np.array(c["contacts"][k], got[k].dtype)), k
    sp = Cg.springs(torch.tensor(c["centroid"], dtype=torch.float64).cuda(), G["p_n"], G["shear_ratio"])
    for k in ("bi", "bj", "pen"):
        assert np.array_equal(sp[k].cpu().numpy(), np.array(c["springs"][k], np.float64 if k == "pen" else np.int32))
    for k in ("e", "g"):
        assert np.array_equal(sp[k].cpu().numpy(), np.array(c["springs"][k], float).reshape(-1, 6)), k


@pytest.mark.parametrize("name,d0", [("tiny", 0.35), ("tiny_shuffled", 0.35), ("ragged_1k", 0.2),
                                     ("ragged_1k", 0.02), ("polygons", 0.15)])
def test_contacts_vs_oracle(dda, name, d0):
    if name == "polygons":
        vptr, vxy, cxy = _random_polygons(600, 3)
    else:
        P = make_slope(preset("tiny", shuffle=True) if name == "tiny_shuffled" else
                       (preset("tiny") if name == "tiny" else preset(1000, seed=1041)))
        vptr, vxy, cxy = _slope_geom(P)
    O = oracle.detect_contacts(vptr, vxy, d0)
    Cg, G = _gpu(dda, vptr, vxy, d0)
    assert O["v"].size > 0
    _same(G, O)
    assert Cg.n_ve == int((O["type"] == 0).sum())
    so = oracle.contact_springs(vptr, vxy, cxy, O, 40.0, 0.4)
    sg = Cg.springs(torch.from_numpy(cxy).cuda(), 40.0, 0.4)
    for k in ("bi", "bj", "pen", "e", "g"):
        assert np.array_equal(sg[k].cpu().numpy(), so[k]), k


def test_contacts_to_solve(dda):
    """Geometry -> contacts -> springs -> K -> BJ-PCG: the detected springs assemble to the same
    matrix as the oracle's springs (bit-exact, O-1) and the solve converges."""
    P = make_slope(preset(1000, seed=1041))
    vptr, vxy, cxy = _slope_geom(P)
    Cg, _ = _gpu(dda, vptr, vxy, 0.2)
    sg = Cg.springs(torch.from_numpy(cxy).cuda(), 40.0, 0.4)
    kd = torch.from_numpy(P.kdiag).cuda()
    K = dda.build_matrix(kd, sg["bi"], sg["bj"], sg["pen"], sg["e"], sg["g"])
    O = oracle.detect_contacts(vptr, vxy, 0.2)
    so = oracle.contact_springs(vptr, vxy, cxy, O, 40.0, 0.4)
    M = oracle.OracleMatrix(P.n, P.kdiag, so["bi"], so["bj"], so["pen"], so["e"], so["g"]).export()
    ex = K.export()
    for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
        assert np.array_equal(ex[k], getattr(M, k)), k
    assert np.array_equal(ex["diag"], M.diag) and np.array_equal(ex["upper"], M.upper)
    d, it, rr, st = K.pcg_solve(torch.from_numpy(P.F).cuda())
    assert st == dda.OK and rr <= 1e-10


@pytest.mark.parametrize("blocks", [10_000, 1_000_000])
def test_contacts_full_size_sampled(dda, blocks):
    """Every record of a sample of vertices (the oracle evaluates one vertex against all edges) at
    the paper-scale and the 1M-block configuration."""
    P = make_slope(preset(blocks, seed=1005 if blocks == 1_000_000 else 1002))
    vptr, vxy, _ = _slope_geom(P)
    d0 = 0.2
    Cg, G = _gpu(dda, vptr, vxy, d0)
    rng = np.random.default_rng(11)
    V = vxy.shape[0]
    sample = np.unique(np.concatenate([[0, V - 1], rng.integers(0, V, 24 if blocks > 100_000 else 200)]))
    for v in sample:
        O = oracle.detect_contacts(vptr, vxy, d0, int(v), int(v) + 1)
        sel = G["v"] == v
        _same({k: G[k][sel] for k in FIELDS}, O)
    assert np.all(np.diff(G["v"].astype(np.int64) * (1 << 32) + G["e"]) > 0)


def test_contacts_bad_input(dda):
    vptr = np.array([0, 2], np.int32)                       # a 2-vertex "polygon"
    vxy = np.zeros((2, 2))
    with pytest.raises(dda.DDAError):
        _gpu(dda, vptr, vxy, 0.1)
    vptr, vxy, _ = _random_polygons(4, 1)
    with pytest.raises(dda.DDAError):
        _gpu(dda, vptr, vxy, 0.0)


def test_contacts_mixed_sizes(dda):
    """One large polygon among small ones: the broad-phase cell is sized by the largest block, so the
    small blocks crowd into few cells — records must still equal the oracle's."""
    vptr, vxy, cxy = _random_polygons(150, 9)
    big = np.array([[3.0, 3.0], [9.0, 3.2], [9.5, 8.0], [3.2, 9.0]])
    vptr2 = np.concatenate([vptr, [vptr[-1] + 4]]).astype(np.int32)
    vxy2 = np.concatenate([vxy, big])
    O = oracle.detect_contacts(vptr2, vxy2, 0.3)
    Cg, G = _gpu(dda, vptr2, vxy2, 0.3)
    assert (O["i"] == 150).any() or (O["j"] == 150).any()
    _same(G, O)


# ------------------------------------------------------------------ second classification (O-10)

ANGLE = os.path.join(os.path.dirname(__file__), "golden", "contact_angle_classes.json")


@pytest.mark.parametrize("case", ["aligned", "corner", "dart"])
def test_classify_golden(dda, case):
    G = json.load(open(ANGLE))
    c = G["cases"][case]
    vptr, vxy = np.array(c["vptr"], np.int32), np.array(c["vxy"], float)
    for tol, want in c["classes"].items():
        Cg, _ = _gpu(dda, vptr, vxy, G["d0"])
        Cg.classify(float(tol))
        got = Cg.export()
        w = np.array(want)
        keep = np.nonzero(w >= 0)[0]
        order = keep[np.argsort(w[keep], kind="stable")]
        assert np.array_equal(got["v"], np.array(c["v"])[order]) and np.array_equal(got["e"], np.array(c["e"])[order])
        assert np.array_equal(got["type"], w[order]), tol
        assert (Cg.n_ve, Cg.n_vv1, Cg.n_vv2) == tuple(int((w == k).sum()) for k in (0, 1, 2))
        if "first_springs" in c and tol == "0.35":
            sp = Cg.springs(torch.tensor(c["centroid"], dtype=torch.float64).cuda(), 3.0, 0.5)
            assert np.array_equal(sp["e"][:2].cpu().numpy(), np.array(c["first_springs"]["e"], float))
            assert np.array_equal(sp["g"][:2].cpu().numpy(), np.array(c["first_springs"]["g"], float))


@pytest.mark.parametrize("name,d0,tol", [("tiny", 0.35, 0.35), ("ragged_1k", 0.2, 0.35), ("polygons", 0.15, 0.35),
                                         ("polygons", 0.15, 0.0), ("polygons", 0.15, 0.8)])
def test_classify_vs_oracle(dda, name, d0, tol):
    """The classified set (records kept by the angle judgment, grouped VE / VV1 / VV2) and the
    springs of every class, bit-exact against O-10 + O-9."""
    if name == "polygons":
        vptr, vxy, cxy = _random_polygons(600, 3)
    else:
        P = make_slope(preset("tiny") if name == "tiny" else preset(1000, seed=1041))
        vptr, vxy, cxy = _slope_geom(P)
    O = oracle.detect_contacts(vptr, vxy, d0)
    Oc = oracle.classified_contacts(vptr, vxy, O, tol)
    Cg, _ = _gpu(dda, vptr, vxy, d0)
    Cg.classify(tol)
    _same(Cg.export(), Oc)
    if name == "polygons" and tol == 0.35:
        assert Cg.n_vv2 > 0 and Cg.n_vv1 > 0 and Cg.count < O["v"].size
    so = oracle.classified_springs(vptr, vxy, cxy, Oc, 40.0, 0.4)
    sg = Cg.springs(torch.from_numpy(cxy).cuda(), 40.0, 0.4)
    for k in ("bi", "bj", "pen", "e", "g"):
        assert np.array_equal(sg[k].cpu().numpy(), so[k]), k


def test_classify_full_size_sampled(dda):
    """1M blocks: the classified records of a vertex sample equal the oracle's classification of that
    vertex's records (the class grouping keeps increasing (v, e) inside each class)."""
    P = make_slope(preset(1_000_000, seed=1005))
    vptr, vxy, cxy = _slope_geom(P)
    Cg, _ = _gpu(dda, vptr, vxy, 0.2)
    n0 = Cg.count
    Cg.classify(0.35)
    G = Cg.export()
    assert Cg.count == Cg.n_ve + Cg.n_vv1 + Cg.n_vv2 and Cg.count < n0
    assert np.all(np.diff(G["type"]) >= 0)
    rng = np.random.default_rng(5)
    V = vxy.shape[0]
    for v in np.unique(np.concatenate([[0, V - 1], rng.integers(0, V, 24)])):
        O = oracle.detect_contacts(vptr, vxy, 0.2, int(v), int(v) + 1)
        Oc = oracle.classified_contacts(vptr, vxy, O, 0.35)
        sel = G["v"] == v
        _same({k: G[k][sel] for k in FIELDS}, Oc)
    sg = Cg.springs(torch.from_numpy(cxy).cuda(), 40.0, 0.4)
    assert sg["bi"].shape[0] == 2 * Cg.count
