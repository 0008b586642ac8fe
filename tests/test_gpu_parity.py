"""GPU parity: the CUDA path through the C ABI vs the oracle.

Bars (BASELINE.json north_star, readings Z8/Z16/Z17):
* structure and index arrays: bit-exact;
* assembled values: bit-exact (both sides round (p*e[r])*g[c] as written);
* SpMV: componentwise |dy_i| <= 1e-12 (|K||x|)_i; unit-vector columns exact;
* PCG: true relative residual <= 1e-10; iterations within max(2, 1%) of the
  oracle; at matched iteration count the solution differs by <= 1e-9 relative.
"""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from synth import make_slope, preset, random_vector, warm_start

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "two_block.json")


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (no CPU fallback exists)")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


CASES = {
    "tiny": lambda: make_slope(preset("tiny")),
    "tiny_shuffled": lambda: make_slope(preset("tiny", shuffle=True)),
    "chain": lambda: make_slope(preset("tiny", courses=1, base_bricks=40)),
    "ragged_1k": lambda: make_slope(preset(1000, seed=1041)),
    "paper": lambda: make_slope(preset("paper")),
}
_cache = {}


def case(name):
    if name not in _cache:
        P = CASES[name]()
        _cache[name] = (P, oracle.assemble(P))
    return _cache[name]


def _abs_bound(O, n, x):
    ip, ix, dv = O.full_csr()
    b = np.zeros(6 * n)
    np.add.at(b, np.repeat(np.arange(6 * n), np.diff(ip)), np.abs(dv) * np.abs(x[ix]))
    return b


# ------------------------------------------------------------------ A1 / A2 assembly

@pytest.mark.parametrize("name", list(CASES))
def test_assembly_bit_exact(dda, name):
    P, O = case(name)
    K = dda.build_from_problem(P)
    S = O.export()
    ex = K.export()
    assert K.n == O.n and K.nnzb == O.nnzb
    for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
        assert np.array_equal(ex[k], getattr(S, k)), k
    assert np.array_equal(ex["diag"], S.diag)
    assert np.array_equal(ex["upper"], S.upper)


def test_golden_two_block(dda):
    G = json.load(open(GOLDEN))
    dev = lambda a, dt: torch.tensor(np.array(a), dtype=dt, device="cuda").contiguous()
    K = dda.build_matrix(dev(G["kdiag"], torch.float64), dev(G["bi"], torch.int32), dev(G["bj"], torch.int32),
                         dev(G["pen"], torch.float64), dev(G["e"], torch.float64), dev(G["g"], torch.float64))
    ex, X = K.export(), G["expect"]
    for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
        assert ex[k].tolist() == X[k], k
    assert np.array_equal(ex["diag"], np.array(X["diag"], float))
    assert np.array_equal(ex["upper"], np.array(X["upper"], float))
    y = K.spmv(dev(X["x"], torch.float64)).cpu().numpy()
    assert np.array_equal(y, np.array(X["y"], float))


def test_no_springs(dda):
    P = make_slope(preset("tiny"))
    dev = "cuda"
    K = dda.build_matrix(torch.from_numpy(P.kdiag).to(dev), torch.zeros(0, dtype=torch.int32, device=dev),
                         torch.zeros(0, dtype=torch.int32, device=dev), torch.zeros(0, dtype=torch.float64, device=dev),
                         torch.zeros((0, 6), dtype=torch.float64, device=dev),
                         torch.zeros((0, 6), dtype=torch.float64, device=dev))
    assert K.nnzb == 0
    ex = K.export()
    U = np.triu(P.kdiag)
    assert np.array_equal(ex["diag"], U + np.transpose(np.triu(U, 1), (0, 2, 1)))
    d, it, rr, st = K.pcg_solve(torch.from_numpy(P.F).cuda(), tol=1e-10)
    assert st == dda.OK and it == 1 and rr <= 1e-10       # block diagonal: BJ is exact


@pytest.mark.parametrize("bad", ["self", "range", "neg_pen", "nan_pen"])
def test_invalid_input(dda, bad):
    P = make_slope(preset("tiny"))
    t = dda.problem_to_device(P)
    if bad == "self":
        t["bj"][3] = t["bi"][3]
    elif bad == "range":
        t["bi"][5] = P.n
    elif bad == "neg_pen":
        t["pen"][7] = -1.0
    else:
        t["pen"][7] = float("nan")
    with pytest.raises(dda.DDAError) as ei:
        dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    assert ei.value.status == dda.ERR_ARG


@pytest.mark.parametrize("name", ["tiny", "paper"])
def test_update_values_matches_fresh_build(dda, name):
    P, _ = case(name)
    t = dda.problem_to_device(P)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    rng = np.random.default_rng(5)
    pen2 = P.pen * rng.uniform(0.5, 1.5, P.m)
    pen2[::7] = 0.0                                      # contacts opened in the open-close loop
    kd2 = P.kdiag * 1.1
    K.update_values(torch.from_numpy(kd2).cuda(), torch.from_numpy(pen2).cuda(), t["e"], t["g"])
    O2 = oracle.OracleMatrix(P.n, kd2, P.bi, P.bj, pen2, P.e, P.g)
    ex, S2 = K.export(), O2.export()
    assert np.array_equal(ex["diag"], S2.diag) and np.array_equal(ex["upper"], S2.upper)


# ------------------------------------------------------------------ A4 SpMV

@pytest.mark.parametrize("name", list(CASES))
def test_spmv_parity(dda, name):
    P, O = case(name)
    K = dda.build_from_problem(P)
    x = random_vector(P.n, 42)
    y = K.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    yo = O.spmv(x)
    bound = _abs_bound(O, P.n, x)
    err = np.abs(y - yo) / bound
    assert err.max() <= 1e-12, err.max()
    assert np.linalg.norm(y - yo) / np.linalg.norm(yo) <= 1e-13


@pytest.mark.parametrize("name", ["tiny", "tiny_shuffled", "ragged_1k"])
def test_spmv_full_storage(dda, name):
    # configs[3] comparison path: the same product from the expanded full-storage BSR6
    P, O = case(name)
    K = dda.build_from_problem(P)
    x = torch.from_numpy(random_vector(P.n, 5)).cuda()
    yf = K.spmv_full(x).cpu().numpy()
    yo = O.spmv(x.cpu().numpy())
    bound = _abs_bound(O, P.n, x.cpu().numpy())
    assert (np.abs(yf - yo) <= 1e-12 * bound).all()


def test_spmv_unit_vectors_exact(dda):
    P, O = case("tiny")
    K = dda.build_from_problem(P)
    ip, ix, dv = O.full_csr()
    import scipy.sparse as sp
    A = sp.csr_matrix((dv, ix, ip), shape=(6 * P.n,) * 2).toarray()
    for k in [0, 1, 5, 6, 100, 6 * P.n // 2, 6 * P.n - 1]:
        x = torch.zeros(6 * P.n, dtype=torch.float64, device="cuda")
        x[k] = 1.0
        assert np.array_equal(K.spmv(x).cpu().numpy(), A[:, k]), k


@pytest.mark.parametrize("name", ["tiny", "tiny_shuffled", "ragged_1k", "paper"])
def test_spmv_tma_ablation_bit_identical(dda, name, monkeypatch):
    """The TMA-staged SpMV ablation (spmv_tma.cu: bulk copies of each 40-row tile's diagonal and
    forward blocks into shared memory, DDA_SPMV_TMA=1) does the default kernel's arithmetic in the same
    order: y bit-identical, including rows whose blocks fall outside the staged ranges (shuffled)."""
    P, O = case(name)
    K = dda.build_from_problem(P)
    x = torch.from_numpy(random_vector(P.n, 5)).cuda()
    monkeypatch.delenv("DDA_SPMV_TMA", raising=False)
    a = K.spmv(x).cpu().numpy()
    monkeypatch.setenv("DDA_SPMV_TMA", "1")
    b = K.spmv(x).cpu().numpy()
    assert np.array_equal(a, b)


def test_spmv_deterministic(dda):
    P, O = case("paper")
    K = dda.build_from_problem(P)
    x = torch.from_numpy(random_vector(P.n, 3)).cuda()
    a = K.spmv(x).cpu().numpy()
    b = K.spmv(x).cpu().numpy()
    assert np.array_equal(a, b)


# ------------------------------------------------------------------ A3 / A7 preconditioners

@pytest.mark.parametrize("name", ["tiny", "paper"])
def test_bj_inverse(dda, name):
    P, O = case(name)
    K = dda.build_from_problem(P)
    dinv = K.bj_setup(full=True).cpu().numpy()
    ref = O.bj_inv()
    D = O.export().diag
    kappa = np.linalg.cond(D)
    for i in range(P.n):
        assert np.linalg.norm(dinv[i] - ref[i]) <= 1e-13 * kappa[i] * np.linalg.norm(ref[i])


def test_bj_not_spd(dda):
    P = make_slope(preset("tiny"))
    kd = P.kdiag.copy()
    kd[17] = -1e6 * np.eye(6)
    t = dda.problem_to_device(P)
    K = dda.build_matrix(torch.from_numpy(kd).cuda(), t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    with pytest.raises(dda.DDAError) as ei:
        K.bj_setup()
    assert ei.value.status == dda.ERR_NOT_SPD
    d, it, rr, st = None, 0, 0, None
    with pytest.raises(dda.DDAError):
        K.pcg_solve(t["F"])


@pytest.mark.parametrize("pc,omega", [("bj", 1.0), ("ssor_ai", 1.0), ("ssor_ai", 0.8), ("ilu0", 1.0)])
def test_precond_apply(dda, pc, omega):
    P, O = case("paper")
    K = dda.build_from_problem(P)
    r = np.random.default_rng(8).standard_normal(6 * P.n)
    z = K.precond_apply(torch.from_numpy(r).cuda(), pc, omega).cpu().numpy()
    if pc == "bj":
        zo = np.einsum("bij,bj->bi", O.bj_inv(), r.reshape(-1, 6)).ravel()
    elif pc == "ilu0":
        zo = O.ilu0_apply(r)
    else:
        zo = O.ssor_ai_apply(r, omega=omega)
    # ILU(0): GPU upper-only IC(0) form vs the oracle's full-pattern IKJ LU (reading Z15)
    tol = 1e-10 if pc == "ilu0" else 1e-12
    assert np.linalg.norm(z - zo) <= tol * np.linalg.norm(zo)


# ------------------------------------------------------------------ A5 / A6 PCG

def _pcg_parity(dda, P, O, pc, omega=1.0, d0=None, tol=1e-10):
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    d0t = torch.from_numpy(d0).cuda() if d0 is not None else None
    d, it, rr, st = K.pcg_solve(F, d0=d0t, tol=tol, precond=pc, omega=omega)
    assert st == dda.OK and rr <= tol * 1.01, (st, rr)
    do, ito, rro, sto = O.pcg(P.F, d0=d0, tol=tol, precond=pc, omega=omega)
    assert sto == oracle.OK and rro <= tol * 1.01
    assert abs(it - ito) <= max(2, int(0.01 * ito)), (it, ito)
    # matched-iteration comparison (reading Z17)
    dm, itm, _, _ = O.pcg(P.F, d0=d0, tol=1e-300, maxit=it, precond=pc, omega=omega)
    assert itm == it
    d = d.cpu().numpy()
    assert np.linalg.norm(d - dm) / np.linalg.norm(dm) <= 1e-9
    return d, it


def _set_engine(dda, engine, loop=-1):
    import ctypes
    f = dda.lib().dda__set_pcg_engine
    f.argtypes = [ctypes.c_int]
    f(engine)
    g = dda.lib().dda__set_scaled_loop
    g.argtypes = [ctypes.c_int]
    g(loop)


@pytest.fixture(params=["auto", "graph", "persistent", "scaled", "scaled_2phase", "scaled_cg1", "scaled_cluster",
                        "scaled_graph"])
def engine(request, dda, monkeypatch):
    """PCG engine: the CUDA-graph while loop, the persistent cooperative kernel, or the
    block-scaled matrix S K S^T (block-Jacobi only; other preconditioners fall back to
    the graph loop) run by one persistent cooperative kernel ('scaled': the two-phase k_sp_loop
    or the single-reduction k_sp_cg1 by size; '_2phase' / '_cg1' force one) or by the
    CUDA-graph while loop ('scaled_graph') — internal hooks; 'auto' picks by size and
    preconditioner."""
    if request.param in ("scaled_2phase", "scaled_cg1", "scaled_cluster"):
        monkeypatch.setenv("DDA_SCALED_CG1", "0" if request.param == "scaled_2phase" else "1")
        monkeypatch.setenv("DDA_SCALED_CLUSTER", "1" if request.param == "scaled_cluster" else "0")
    _set_engine(dda, *{"auto": (-1, -1), "graph": (0, -1), "persistent": (1, -1), "scaled": (2, 1),
                       "scaled_2phase": (2, 1), "scaled_cg1": (2, 1), "scaled_cluster": (2, 1),
                       "scaled_graph": (2, 0)}[request.param])
    yield request.param
    _set_engine(dda, -1, -1)


@pytest.mark.parametrize("name", ["tiny", "tiny_shuffled", "ragged_1k", "paper"])
def test_pcg_bj(dda, name, engine):
    P, O = case(name)
    _pcg_parity(dda, P, O, "bj")


@pytest.mark.parametrize("name", ["tiny", "paper"])
def test_pcg_ssor_ai(dda, name, engine):
    P, O = case(name)
    _pcg_parity(dda, P, O, "ssor_ai")


@pytest.mark.parametrize("name", ["tiny", "tiny_shuffled", "paper"])
def test_pcg_ilu0(dda, name):
    P, O = case(name)
    _pcg_parity(dda, P, O, "ilu0")


def test_ilu0_chain_exact(dda):
    P, O = case("chain")          # a single course: tridiagonal block pattern, no fill
    K = dda.build_from_problem(P)
    d, it, rr, st = K.pcg_solve(torch.from_numpy(P.F).cuda(), precond="ilu0")
    assert st == dda.OK and it == 1 and rr <= 1e-10


def test_preconditioner_trend(dda):
    # Table I P:173 / P:162: iterations ILU < SSOR-AI < BJ
    P, O = case("paper")
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    its = {pc: K.pcg_solve(F, precond=pc)[1] for pc in ("bj", "ssor_ai", "ilu0")}
    assert its["ilu0"] < its["ssor_ai"] < its["bj"], its


def test_pcg_none(dda, engine):
    P, O = case("tiny")
    _pcg_parity(dda, P, O, "none")


def test_pcg_tiny_vs_dense_ldlt(dda):
    P, O = case("tiny")
    d, _ = _pcg_parity(dda, P, O, "bj")
    ref = O.ldlt_solve(P.F)
    import scipy.linalg as sla
    from conftest import dense_from_springs
    Kd = dense_from_springs(P)
    ev = np.linalg.eigvalsh(Kd)
    assert np.linalg.norm(d - ref) / np.linalg.norm(ref) <= (ev.max() / ev.min()) * 1e-10


def test_pcg_warm_start_and_edge_cases(dda, engine):
    P, O = case("paper")
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    d1, it1, rr1, st1 = K.pcg_solve(F)
    d0 = warm_start(d1.cpu().numpy(), 9)
    _, it2 = _pcg_parity(dda, P, O, "bj", d0=d0)
    assert it2 < it1
    # d0 aliasing d
    dd = torch.from_numpy(d0).cuda()
    _, it3, rr3, st3 = K.pcg_solve(F, d0=dd, d=dd)
    assert st3 == dda.OK and it3 == it2 and rr3 <= 1.01e-10
    # F = 0 -> d = 0, 0 iterations (reading Z2)
    z, itz, rrz, stz = K.pcg_solve(torch.zeros_like(F), d0=torch.ones_like(F))
    assert stz == dda.OK and itz == 0 and rrz == 0.0 and not z.any()
    # iteration cap (the paper's DDA policy caps at 200)
    _, it5, rr5, st5 = K.pcg_solve(F, maxit=200)
    assert st5 == dda.ERR_NO_CONVERGENCE and it5 == 200 and rr5 > 1e-10


@pytest.mark.parametrize("loop", [1, 0], ids=["persistent", "graph"])
def test_scaled_engine_stopping_test(dda, loop):
    """The scaled engine evaluates the exact stopping test |L r~| only when lam |r~|^2 allows it to
    pass: it must stop at the same iteration as the unscaled loop with far fewer
    exact tests than iterations — with either loop driver."""
    P, O = case("paper")
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    try:
        _set_engine(dda, 0)
        d0, it0, rr0, st0 = K.pcg_solve(F)
        _set_engine(dda, 2, loop)
        d2, it2, rr2, st2 = K.pcg_solve(F)
    finally:
        _set_engine(dda, -1, -1)
    assert st0 == st2 == dda.OK
    assert abs(it0 - it2) <= 1, (it0, it2)
    checks = K.last_checks()
    assert 1 <= checks < it2 // 2, (checks, it2)
    assert np.linalg.norm(d2.cpu().numpy() - d0.cpu().numpy()) <= 1e-8 * np.linalg.norm(d0.cpu().numpy())


@pytest.mark.parametrize("cg1", ["0", "1"], ids=["2phase", "cg1"])
@pytest.mark.parametrize("eng", [(-1, -1), (2, 1), (2, 0)], ids=["auto", "scaled", "scaled_graph"])
def test_pcg_deterministic(dda, eng, cg1, monkeypatch):
    monkeypatch.setenv("DDA_SCALED_CG1", cg1)
    P, O = case("paper")
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    try:
        _set_engine(dda, *eng)
        a = K.pcg_solve(F)[0].cpu().numpy()
        b = K.pcg_solve(F)[0].cpu().numpy()
    finally:
        _set_engine(dda, -1, -1)
    assert np.array_equal(a, b)


def test_scaled_loops_agree(dda):
    """The persistent and the CUDA-graph drivers of the scaled engine run the same iteration; only
    the CTA count of the r~ update (hence the rounding of one dot product) differs."""
    P, O = case("paper")
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    out = {}
    try:
        for loop in (1, 0):
            _set_engine(dda, 2, loop)
            d, it, rr, st = K.pcg_solve(F)
            out[loop] = (d.cpu().numpy(), it, rr, st, K.last_checks())
    finally:
        _set_engine(dda, -1, -1)
    (dp, itp, rrp, stp, cp), (dg, itg, rrg, stg, cg) = out[1], out[0]
    assert stp == stg == dda.OK and abs(itp - itg) <= 1 and rrp <= 1e-10 and rrg <= 1e-10
    assert np.linalg.norm(dp - dg) <= 1e-9 * np.linalg.norm(dg)


@pytest.mark.parametrize("name", ["paper", "ragged_1k"])
def test_single_reduction_loop_matches_two_phase(dda, name, monkeypatch):
    """k_sp_cg1 (Chronopoulos-Gear: s = Ks r carried, one grid barrier per iteration) runs the same
    Krylov iterates as k_sp_loop in exact arithmetic: same stopping iteration (+-1), solutions
    within the PCG tolerance, and each matches the oracle at the matched iteration (reading Z17)."""
    P, O = case(name)
    out = {}
    try:
        _set_engine(dda, 2, 1)
        for v in ("0", "1"):
            monkeypatch.setenv("DDA_SCALED_CG1", v)
            out[v] = _pcg_parity(dda, P, O, "bj")
    finally:
        _set_engine(dda, -1, -1)
    (d0, it0), (d1, it1) = out["0"], out["1"]
    assert abs(it0 - it1) <= 1, (it0, it1)
    assert np.linalg.norm(d1 - d0) <= 1e-9 * np.linalg.norm(d0)


def test_solve_host_e2e(dda):
    P, O = case("paper")
    d, it, rr, st = dda.solve_host(P.kdiag, P.bi, P.bj, P.pen, P.e, P.g, P.F)
    K = dda.build_from_problem(P)
    d2, it2, rr2, st2 = K.pcg_solve(torch.from_numpy(P.F).cuda())
    assert st == st2 == dda.OK and it == it2
    assert np.array_equal(d, d2.cpu().numpy())


@pytest.mark.parametrize("loop", ["2phase", "cg1", "graph"])
def test_residual_history(dda, loop, monkeypatch):
    """dda_pcg_set_history: per iteration rho_{k+1} = r^T M^-1 r and, where the exact stopping test
    ran, |r|^2.  rho_k is checked against r_k = F - K d_k recomputed from a maxit = k solve (d_k from
    the same engine; r^T D^-1 r through dda_precond_apply); the exact entries against the reported
    true residual at the stop; entries past the last iteration stay untouched."""
    monkeypatch.setenv("DDA_SCALED_CG1", "1" if loop == "cg1" else "0")
    P, O = case("paper")
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    try:
        _set_engine(dda, 2, 0 if loop == "graph" else 1)
        hist = torch.full((400, 2), -1.0, dtype=torch.float64, device="cuda")
        K.set_history(hist)
        d, it, rr, st = K.pcg_solve(F)
        h = hist.cpu().numpy()
        assert st == dda.OK and 0 < it < 400
        assert np.all(np.isfinite(h[:it, 0])) and np.all(h[:it, 0] > 0) and np.all(h[it:] == -1.0)
        exact = ~np.isnan(h[:it, 1])
        assert exact.sum() == K.last_checks() and exact[it - 1]
        fn = float(np.linalg.norm(P.F))
        assert abs(np.sqrt(h[it - 1, 1]) / fn - rr) <= 1e-3 * rr          # recursive vs true residual at the stop
        assert np.sqrt(h[it - 1, 1]) <= 1e-10 * fn
        for k in (1, 5, 20):
            dk, itk, _, _ = K.pcg_solve(F, tol=1e-300, maxit=k)
            r = F - K.spmv(dk)
            rho = float(torch.dot(r, K.precond_apply(r, precond="bj")))
            assert abs(hist[k - 1, 0].item() - rho) <= 1e-8 * rho, (k, hist[k - 1, 0].item(), rho)
        K.set_history(None)
        hist.fill_(-1.0)
        K.pcg_solve(F)
        assert bool((hist == -1.0).all())
    finally:
        _set_engine(dda, -1, -1)


@pytest.mark.parametrize("pc", ["bj", "ssor_ai"])
def test_cooperative_fallback(dda, pc, monkeypatch):
    """When not even one CTA of the persistent kernel fits per SM (DDA_SIMULATE_NO_COOP stands in for a
    caller context with a smaller shared-memory carve-out), the solve falls back before writing any
    state: scaled BJ to the CUDA-graph while loop, SSOR-AI to the unscaled graph engine.  Same stop
    rule; parity against the oracle (Z17)."""
    P, O = case("paper")
    monkeypatch.setenv("DDA_SIMULATE_NO_COOP", "1")
    d, it = _pcg_parity(dda, P, O, pc)
    monkeypatch.delenv("DDA_SIMULATE_NO_COOP")
    d2, it2 = _pcg_parity(dda, P, O, pc)
    assert abs(it - it2) <= 1 and np.linalg.norm(d - d2) <= 1e-9 * np.linalg.norm(d2)


def test_solve_host_batch(dda):
    """Streamed batch (dda_solve_host_batch): systems of different sizes, one with a warm start and
    one repeated (so both input slots are refilled), each bit-identical to dda_solve_host; pinned and
    pageable host buffers."""
    names = ["paper", "tiny", "paper", "ragged_1k", "tiny"]
    systems, refs = [], []
    for k, name in enumerate(names):
        P, O = case(name)
        pin = (lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()) if k % 2 == 0 else (lambda a: a)
        S = {f: pin(getattr(P, f)) for f in ("kdiag", "bi", "bj", "pen", "e", "g", "F")}
        d0 = warm_start(np.zeros(6 * P.n), 3) if k == 2 else None
        if d0 is not None:
            S["d0"] = pin(d0)
        S["d"] = pin(np.full(6 * P.n, np.nan))
        systems.append(S)
        refs.append(dda.solve_host(P.kdiag, P.bi, P.bj, P.pen, P.e, P.g, P.F, d0=d0))
    out = dda.solve_host_batch(systems)
    for S, (dr, itr, rrr, str_), (it, rr, st) in zip(systems, refs, out):
        d = S["d"].numpy() if hasattr(S["d"], "numpy") else S["d"]
        assert st == str_ == dda.OK and it == itr and rr == rrr
        assert np.array_equal(d, dr)
    assert dda.solve_host_batch([]) == []


@pytest.mark.parametrize("name", ["tiny", "paper"])
def test_scaled_ssor_omega0_is_bj(dda, name):
    """SSOR-AI with omega = 0 is M^{-1} = D^{-1} (reading Z14): the scaled SSOR-AI kernel must take the
    iterations of block-Jacobi and reach the same solution."""
    P, O = case(name)
    K = dda.build_from_problem(P)
    F = torch.from_numpy(P.F).cuda()
    try:
        _set_engine(dda, 2, 1)
        db, itb, rrb, stb = K.pcg_solve(F, precond="bj")
        ds, its, rrs, sts = K.pcg_solve(F, precond="ssor_ai", omega=0.0)
    finally:
        _set_engine(dda, -1, -1)
    assert stb == sts == dda.OK and itb == its, (itb, its)
    db, ds = db.cpu().numpy(), ds.cpu().numpy()
    assert np.linalg.norm(ds - db) <= 1e-12 * np.linalg.norm(db)


def test_new_entry_points_reject_bad_arguments(dda):
    """Argument checks of the round-2 entry points (dda.h): dda_pcg_set_history with a buffer / capacity
    mismatch, dda_solve_host_batch with a system missing its arrays, and the IPC import of blobs that
    are not a consistent set (wrong size, wrong rank order) or on a communicator without a partition."""
    import ctypes as C
    L = dda.lib()
    P, O = case("tiny")
    K = dda.build_from_problem(P)
    assert L.dda_pcg_set_history(K.handle, None, 5) == dda.ERR_ARG
    assert L.dda_pcg_set_history(None, None, 0) == dda.ERR_ARG
    assert L.dda_pcg_set_history(K.handle, None, 0) == dda.OK
    bad = (dda.HostSystem * 1)()
    bad[0].n_blocks = P.n
    assert L.dda_solve_host_batch(1, bad, 1e-10, 100, 0, 1.0, None) == dda.ERR_ARG
    assert L.dda_solve_host_batch(-1, None, 1e-10, 100, 0, 1.0, None) == dda.ERR_ARG
    assert L.dda_solve_host_batch(0, None, 1e-10, 100, 0, 1.0, None) == dda.OK
    # IPC: import before a partition exists, then blobs of the wrong size / order
    c = dda.Comm.ipc(2, 0)
    n = C.c_int64()
    assert L.dda_comm_ipc_export(c._h, None, C.byref(n)) == dda.OK and n.value > 0
    buf = C.create_string_buffer(2 * n.value)
    assert L.dda_comm_ipc_import(c._h, buf, n.value) == dda.ERR_ARG         # no partition attached
    t = dda.problem_to_device(P)
    b = dda.row_bounds(P.n, 2)
    c.build_matrix_dist(0, P.n, b, t["kdiag"][: int(b[1])].contiguous(), t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    blob = c.ipc_export()
    assert L.dda_comm_ipc_import(c._h, C.create_string_buffer(blob * 2, 2 * len(blob)), len(blob) - 8) == dda.ERR_ARG
    assert L.dda_comm_ipc_import(c._h, C.create_string_buffer(blob * 2, 2 * len(blob)), len(blob)) == dda.ERR_ARG   # rank 0 twice
    c.free()
    with pytest.raises(Exception):
        dda.Comm.ipc(2, 5)


@pytest.mark.parametrize("sync,discard", [("0", "1"), ("0", "0"), ("1", "1"), ("3", "0")],
                         ids=["flags", "flags_keep", "step_counters", "parity_tags"])
@pytest.mark.parametrize("name", ["tiny", "ragged_1k", "paper"])
def test_push_form_phase_a(dda, name, sync, discard, monkeypatch):
    """The opt-in push form of k_sp_loop's phase A (phase_a_lr: each upper block applied once in both
    directions, V_ij^T p_i pushed to an L2-resident entry the row j sums; the paper's up-res / low-res
    scheme, in one sweep) under each ordering of pushes before reads: oracle parity
    (reading Z17), bitwise repeatability, and agreement with the pull form."""
    P, O = case(name)
    monkeypatch.setenv("DDA_SCALED_CG1", "0")
    out = {}
    try:
        _set_engine(dda, 2, 1)
        monkeypatch.setenv("DDA_SP_LR", "0")
        out["pull"] = _pcg_parity(dda, P, O, "bj")
        monkeypatch.setenv("DDA_SP_LR", "1")
        monkeypatch.setenv("DDA_LR_SYNC", sync)
        monkeypatch.setenv("DDA_LR_DISCARD", discard)
        out["push"] = _pcg_parity(dda, P, O, "bj")
        K = dda.build_from_problem(P)
        F = torch.from_numpy(P.F).cuda()
        a = K.pcg_solve(F)[0].cpu().numpy()
        b = K.pcg_solve(F)[0].cpu().numpy()
    finally:
        _set_engine(dda, -1, -1)
    assert np.array_equal(a, b)
    (dl, itl), (dp, itp) = out["pull"], out["push"]
    assert abs(itl - itp) <= 1, (itl, itp)
    assert np.linalg.norm(dp - dl) <= 1e-9 * np.linalg.norm(dl)
