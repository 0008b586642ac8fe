"""NEXT-4 GPU parity: the interpenetration check / open-close switch (dda_contact_check), the gap
load (dda_contact_loads) and the open-close loop (dda_open_close) against the oracle's O-11 / O-12
and its loop, through the C ABI.  States, categories, penalties and loads bit-exact for the same
solution d; the loop's final states equal the oracle loop's, its solution within the bound the
two 1e-10 solves allow (2 kappa 1e-10 <= 1e-7, kappa ~ 500)."""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from synth import make_slope, preset, random_vector

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "contact_states.json")
P_N, SR, TPHI, OTOL, STOL = 40.0, 0.4, 0.577, 0.01, 0.35


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (no CPU fallback exists)")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


def _gpu_set(dda, vptr, vxy, cxy, d0, stol, p_n, sr):
    Cg = dda.detect_contacts(torch.from_numpy(vptr).cuda(), torch.from_numpy(np.ascontiguousarray(vxy)).cuda(), d0)
    Cg.classify(stol)
    sp = Cg.springs(torch.from_numpy(np.ascontiguousarray(cxy)).cuda(), p_n, sr)
    return Cg, sp


@pytest.mark.parametrize("case", ["offset", "corner"])
def test_golden_checks(dda, case):
    G = json.load(open(GOLDEN))
    c = G[case]
    vptr, vxy, cxy = np.array(c["vptr"], np.int32), np.array(c["vxy"], float), np.array(c["centroid"], float)
    Cg, sp = _gpu_set(dda, vptr, vxy, cxy, G["d0"], G["sin_tol"], G["p_n"], G["shear_ratio"])
    st0 = Cg.init_states()
    if "state0" in c:
        assert np.array_equal(st0.cpu().numpy(), c["state0"])
        pen = torch.tensor([3.0, 1.5, 3.0, 1.5], dtype=torch.float64, device="cuda")
        assert np.array_equal(Cg.loads(sp, pen).cpu().numpy(), c["Fc_closed"])
    for name, ck in c["checks"].items():
        d = torch.zeros(12, dtype=torch.float64, device="cuda")
        d[6:8] = torch.tensor(ck["dB"], dtype=torch.float64)
        state = torch.tensor(ck["old"], dtype=torch.int32, device="cuda")
        pen, cat, order, counts = Cg.check(d, sp, state, G["p_n"], G["shear_ratio"], G["tan_phi"], G["open_tol"])
        assert np.array_equal(state.cpu().numpy(), ck["state"]), name
        assert np.array_equal(cat.cpu().numpy(), ck["cat"]), name
        assert np.array_equal(pen.cpu().numpy(), ck["pen"]), name
        assert np.array_equal(counts, np.bincount(ck["cat"], minlength=6)), name


def _slope(n=None, seed=1041):
    P = make_slope(preset("tiny") if n is None else preset(n, seed=seed))
    vptr = (4 * np.arange(P.n + 1)).astype(np.int32)
    vxy = P.verts.reshape(-1, 2).copy()
    V = P.verts
    area = 0.5 * np.abs(np.sum(V[:, :, 0] * np.roll(V[:, :, 1], -1, 1) - np.roll(V[:, :, 0], -1, 1) * V[:, :, 1], 1))
    F = np.zeros((P.n, 6))
    F[:, 1] = -area
    return P, vptr, vxy, F.reshape(-1)


@pytest.mark.parametrize("n", [None, 1000])
def test_check_and_loads_vs_oracle(dda, n):
    """Same d and old states on both sides: states, categories, penalties, category order and the
    gap load bit-exact."""
    P, vptr, vxy, F = _slope(n)
    Cg, sp = _gpu_set(dda, vptr, vxy, P.centroid, 0.35, STOL, P_N, SR)
    O = oracle.detect_contacts(vptr, vxy, 0.35)
    Oc = oracle.classified_contacts(vptr, vxy, O, STOL)
    so = oracle.classified_springs(vptr, vxy, P.centroid, Oc, P_N, SR)
    st0 = Cg.init_states()
    Fo, sto = oracle.contact_loads(P.n, vptr, vxy, Oc, so["e"], so["g"], None)
    assert np.array_equal(st0.cpu().numpy(), sto)
    rng = np.random.default_rng(3)
    old = rng.integers(0, 3, Oc["i"].size).astype(np.int32)
    pen_o = oracle.state_penalties(old, P_N, SR)
    Fo, _ = oracle.contact_loads(P.n, vptr, vxy, Oc, so["e"], so["g"], pen_o)
    Fg = Cg.loads(sp, torch.from_numpy(pen_o).cuda(), torch.from_numpy(F).cuda()).cpu().numpy()
    assert np.array_equal(Fg, F + Fo)
    d = 0.02 * random_vector(P.n, 9)
    so_st, so_cat, so_pen = oracle.contact_check(vptr, vxy, Oc, d, so["e"], so["g"], P_N, SR, TPHI, OTOL, old)
    state = torch.from_numpy(old.copy()).cuda()
    pen, cat, order, counts = Cg.check(torch.from_numpy(d).cuda(), sp, state, P_N, SR, TPHI, OTOL)
    assert np.array_equal(state.cpu().numpy(), so_st)
    assert np.array_equal(cat.cpu().numpy(), so_cat)
    assert np.array_equal(pen.cpu().numpy(), so_pen)
    assert np.array_equal(order.cpu().numpy(), np.argsort(so_cat, kind="stable"))
    assert np.array_equal(counts, np.bincount(so_cat, minlength=6))
    assert counts[1] > 0 and counts[2] > 0 and counts[3] > 0


@pytest.mark.parametrize("n", [None, 1000])
def test_open_close_loop_vs_oracle(dda, n):
    """Loop 3 on the GPU (dda_open_close) against the oracle's loop: same number of open-close
    iterations, identical final states, solutions within the bound of two 1e-10 solves."""
    P, vptr, vxy, F = _slope(n)
    O = oracle.detect_contacts(vptr, vxy, 0.35)
    Oc = oracle.classified_contacts(vptr, vxy, O, STOL)
    do, sto, hist, conv_o = oracle.open_close_loop(P.n, P.kdiag, F, vptr, vxy, P.centroid, Oc, P_N, SR, TPHI, OTOL)
    assert conv_o
    Cg, sp = _gpu_set(dda, vptr, vxy, P.centroid, 0.35, STOL, P_N, SR)
    state = Cg.init_states()
    kd = torch.from_numpy(P.kdiag).cuda()
    K = dda.build_matrix(kd, sp["bi"], sp["bj"], sp["pen"], sp["e"], sp["g"])
    Fd = torch.from_numpy(F).cuda()
    d, state, pen, oc, pit, conv, rr = Cg.open_close(K, kd, Fd, sp, state, p_n=P_N, shear_ratio=SR, tan_phi=TPHI,
                                                     open_tol=OTOL)
    assert conv and oc == len(hist)
    assert np.array_equal(state.cpu().numpy(), sto)
    assert rr <= 1.01e-10
    dg = d.cpu().numpy()
    assert np.linalg.norm(dg - do) <= 1e-7 * np.linalg.norm(do)
    # the GPU solution solves the oracle's final system (its states' matrix and loads)
    so = oracle.classified_springs(vptr, vxy, P.centroid, Oc, P_N, SR)
    pen_o = oracle.state_penalties(sto, P_N, SR)
    assert np.array_equal(pen.cpu().numpy(), pen_o)
    M = oracle.OracleMatrix(P.n, P.kdiag, so["bi"], so["bj"], pen_o, so["e"], so["g"])
    Fc, _ = oracle.contact_loads(P.n, vptr, vxy, Oc, so["e"], so["g"], pen_o)
    res = F + Fc - M.spmv(dg)
    assert np.linalg.norm(res) <= 1.05e-10 * np.linalg.norm(F + Fc)


def test_check_full_size_sampled(dda):
    """1M blocks: the check and the gap load on a sample of contacts / blocks against O-11 / O-12
    evaluated on those records only."""
    P = make_slope(preset(1_000_000, seed=1005))
    vptr = (4 * np.arange(P.n + 1)).astype(np.int32)
    vxy = P.verts.reshape(-1, 2).copy()
    Cg, sp = _gpu_set(dda, vptr, vxy, P.centroid, 0.2, STOL, P_N, SR)
    st0 = Cg.init_states()
    G = Cg.export()
    m = Cg.count
    rng = np.random.default_rng(8)
    old = rng.integers(0, 3, m).astype(np.int32)
    d = 0.02 * random_vector(P.n, 10)
    state = torch.from_numpy(old.copy()).cuda()
    pen, cat, order, counts = Cg.check(torch.from_numpy(d).cuda(), sp, state, P_N, SR, TPHI, OTOL)
    e, g = sp["e"].cpu().numpy(), sp["g"].cpu().numpy()
    ks = np.unique(np.concatenate([[0, m - 1], rng.integers(0, m, 20000)]))
    sub = {k: G[k][ks] for k in ("i", "v", "j", "e", "type")}
    rows = np.stack([2 * ks, 2 * ks + 1], 1).reshape(-1)
    s_st, s_cat, s_pen = oracle.contact_check(vptr, vxy, sub, d, e[rows], g[rows], P_N, SR, TPHI, OTOL, old[ks])
    assert np.array_equal(state.cpu().numpy()[ks], s_st)
    assert np.array_equal(cat.cpu().numpy()[ks], s_cat)
    assert np.array_equal(pen.cpu().numpy()[rows], s_pen)
    _, s_st0 = oracle.contact_loads(P.n, vptr, vxy, sub, e[rows], g[rows], None)
    assert np.array_equal(st0.cpu().numpy()[ks], s_st0)
    # gap load of sampled blocks: every contact touching them
    blocks = np.unique(rng.integers(0, P.n, 2000))
    touch = np.nonzero(np.isin(G["i"], blocks) | np.isin(G["j"], blocks))[0]
    sub = {k: G[k][touch] for k in ("i", "v", "j", "e", "type")}
    rows = np.stack([2 * touch, 2 * touch + 1], 1).reshape(-1)
    pen_all = oracle.state_penalties(old, P_N, SR)
    Fo, _ = oracle.contact_loads(P.n, vptr, vxy, sub, e[rows], g[rows], pen_all[rows])
    Fg = Cg.loads(sp, torch.from_numpy(pen_all).cuda()).cpu().numpy()
    idx = (6 * blocks[:, None] + np.arange(6)).reshape(-1)
    assert np.array_equal(Fg[idx], Fo[idx])


def test_contact_transfer_vs_oracle(dda):
    """NEXT-3 contact transfer: states of a perturbed next step (contacts within 0.35 h) from the
    previous step's converged states (contacts within 0.1 h), against O-13, bit-exact, matched count."""
    P, vptr, vxy, F = _slope(1000)
    Cg, sp = _gpu_set(dda, vptr, vxy, P.centroid, 0.1, STOL, P_N, SR)
    state = Cg.init_states()
    kd = torch.from_numpy(P.kdiag).cuda()
    K = dda.build_matrix(kd, sp["bi"], sp["bj"], sp["pen"], sp["e"], sp["g"])
    _, state, _, oc, _, conv, _ = Cg.open_close(K, kd, torch.from_numpy(F).cuda(), sp, state, p_n=P_N,
                                                shear_ratio=SR, tan_phi=TPHI, open_tol=OTOL)
    assert conv
    rng = np.random.default_rng(3)
    vxy2 = vxy + rng.uniform(-0.05, 0.05, vxy.shape)
    C2, sp2 = _gpu_set(dda, vptr, vxy2, P.centroid, 0.35, STOL, P_N, SR)
    st2 = C2.init_states()
    init = st2.cpu().numpy().copy()
    matched = C2.transfer_from(Cg, state, st2)
    O1, O2 = Cg.export(), C2.export()
    want, mo = oracle.contact_transfer(O1, state.cpu().numpy(), O2, init)
    assert np.array_equal(st2.cpu().numpy(), want) and matched == mo
    assert 0 < matched < C2.count
