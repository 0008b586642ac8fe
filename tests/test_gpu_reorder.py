"""NEXT-2 on the GPU: dda_build_matrix_reordered (internal RCM order, the caller's numbering at
every entry point) against the oracle, through the C ABI: the export in the caller's numbering
bit-exact (structure and values, O-1), SpMV <= 1e-12 componentwise, D^{-1} and the preconditioner
applies in the caller's numbering, PCG per Z17, value-only re-assembly bit-exact; and on a shuffled
numbering at size the reordered SpMV is faster than the plain one (the L2 reuse it restores)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from synth import make_slope, preset, random_vector

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (no CPU fallback exists)")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


@pytest.fixture(scope="module", params=["tiny_shuffled", "shuffled_5k"])
def case(request, dda):
    P = make_slope(preset("tiny", shuffle=True) if request.param == "tiny_shuffled"
                   else preset(5000, seed=1050, shuffle=True))
    O = oracle.assemble(P)
    t = dda.problem_to_device(P)
    K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"], reorder=True)
    return P, O, t, K


def test_export_in_caller_numbering_bit_exact(dda, case):
    P, O, t, K = case
    S, ex = O.export(), K.export()
    for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
        assert np.array_equal(ex[k], getattr(S, k)), k
    assert np.array_equal(ex["diag"], S.diag) and np.array_equal(ex["upper"], S.upper)


def test_spmv_and_precond(dda, case):
    P, O, t, K = case
    x = random_vector(P.n, 21)
    y = K.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    yo = O.spmv(x)
    ip, ix, dv = O.full_csr()
    bound = np.zeros(6 * P.n)
    np.add.at(bound, np.repeat(np.arange(6 * P.n), np.diff(ip)), np.abs(dv) * np.abs(x[ix]))
    assert (np.abs(y - yo) <= 1e-12 * bound).all()
    yf = K.spmv_full(torch.from_numpy(x).cuda()).cpu().numpy()
    assert (np.abs(yf - yo) <= 1e-12 * bound).all()
    dinv = K.bj_setup(full=True).cpu().numpy()
    ref = O.bj_inv()
    kappa = np.linalg.cond(O.export().diag)
    assert all(np.linalg.norm(dinv[i] - ref[i]) <= 1e-13 * kappa[i] * np.linalg.norm(ref[i]) for i in range(P.n))
    z = K.precond_apply(torch.from_numpy(x).cuda(), "bj").cpu().numpy()
    zo = np.einsum("bij,bj->bi", ref, x.reshape(-1, 6)).ravel()
    assert np.linalg.norm(z - zo) <= 1e-12 * np.linalg.norm(zo)


@pytest.mark.parametrize("pc", ["bj", "ssor_ai", "ilu0"])
def test_pcg_z17(dda, case, pc):
    P, O, t, K = case
    d, it, rr, st = K.pcg_solve(t["F"], tol=1e-10, precond=pc)
    assert st == dda.OK and rr <= 1.01e-10
    res = P.F - O.spmv(d.cpu().numpy())
    assert np.linalg.norm(res) <= 1.05e-10 * np.linalg.norm(P.F)        # the caller's system, by the oracle
    if pc != "bj":
        # SSOR-AI's triangular split and ILU(0)'s incomplete factor depend on the block order: on a
        # reordered matrix they are those of the internal (RCM) order, so only convergence is compared
        return
    do, ito, _, _ = O.pcg(P.F, tol=1e-10, precond=pc)
    assert abs(it - ito) <= max(2, int(0.01 * ito)), (it, ito)
    dm, _, _, _ = O.pcg(P.F, tol=1e-300, maxit=it, precond=pc)
    assert np.linalg.norm(d.cpu().numpy() - dm) <= 1e-9 * np.linalg.norm(dm)


def test_update_values(dda, case):
    P, O, t, K = case
    rng = np.random.default_rng(4)
    pen2 = P.pen * rng.uniform(0.5, 1.5, P.m)
    kd2 = P.kdiag * 1.07
    K2 = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"], reorder=True)
    K2.update_values(torch.from_numpy(kd2).cuda(), torch.from_numpy(pen2).cuda(), t["e"], t["g"])
    S2 = oracle.OracleMatrix(P.n, kd2, P.bi, P.bj, pen2, P.e, P.g).export()
    ex = K2.export()
    assert np.array_equal(ex["diag"], S2.diag) and np.array_equal(ex["upper"], S2.upper)


def test_reordered_spmv_faster_on_shuffled_numbering(dda):
    """256k blocks (the matrix is 2.6x L2), randomly numbered: the internal RCM order restores the L2
    reuse of the transposed re-reads (vector permutations included in the timed call)."""
    P = make_slope(preset(262_144, seed=1047, shuffle=True))
    t = dda.problem_to_device(P)
    Kp = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    Kr = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"], reorder=True)
    x = torch.rand(6 * P.n, dtype=torch.float64, device="cuda")
    ms = {}
    for name, K in (("plain", Kp), ("reordered", Kr)):
        y = torch.empty_like(x)
        for _ in range(3):
            K.spmv(x, y)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(10):
            K.spmv(x, y)
        b.record()
        torch.cuda.synchronize()
        ms[name] = a.elapsed_time(b) / 10
    assert torch.allclose(Kp.spmv(x), Kr.spmv(x), rtol=1e-12, atol=1e-12)
    assert ms["reordered"] < ms["plain"], ms
