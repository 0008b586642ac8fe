"""GPU parity of the block-row partitioned solver (§8(e)) through the C ABI.

Only one GPU is available to the test run, so the partitioned algorithm is
exercised with the LOOPBACK transport (P partitions in one process, halo by
device copy, allreduce as an ordered host sum) and the NCCL transport with a
single rank; multi-rank NCCL runs in bench.py under torchrun on a multi-GPU box.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from paper_conf_ipps_xiaohmxw17_b200.partition import row_bounds, local_from_slope
from synth import make_slope, preset, random_vector

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


@pytest.fixture(scope="module")
def prob():
    P = make_slope(preset(20_000, seed=1043))
    return P, oracle.assemble(P)


def _setup(dda, P, nparts):
    b = row_bounds(P.n, nparts)
    comm = dda.Comm.loopback(nparts)
    lps, Ks = [], []
    for r in range(nparts):
        lp = local_from_slope(P, b, r)
        K = dda.build_local(lp)
        comm.attach(r, K, lp)
        lps.append(lp); Ks.append(K)
    return comm, lps, Ks


@pytest.mark.parametrize("nparts", [1, 2, 3, 4])
def test_spmv_dist_loopback(dda, prob, nparts):
    P, O = prob
    comm, lps, Ks = _setup(dda, P, nparts)
    x = random_vector(P.n, 11)
    xs = [torch.from_numpy(x[6 * lp.r0: 6 * lp.r1].copy()).cuda() for lp in lps]
    ys = comm.spmv(xs)
    y = np.concatenate([t.cpu().numpy() for t in ys])
    yo = O.spmv(x)
    ip, ix, dv = O.full_csr()
    bound = np.zeros(6 * P.n)
    np.add.at(bound, np.repeat(np.arange(6 * P.n), np.diff(ip)), np.abs(dv) * np.abs(x[ix]))
    assert (np.abs(y - yo) <= 1e-12 * bound).all()


@pytest.fixture(params=["v3", "v2"])
def dist_version(request, monkeypatch):
    """v3 = the scaled block-Jacobi engine per partition (default); v2 = the unscaled loop
    (DDA_DIST_SCALED=0, read by the library on every solve)."""
    if request.param == "v2":
        monkeypatch.setenv("DDA_DIST_SCALED", "0")
    else:
        monkeypatch.delenv("DDA_DIST_SCALED", raising=False)
    return request.param


@pytest.mark.parametrize("nparts", [1, 2, 4])
def test_pcg_dist_loopback(dda, prob, nparts, dist_version):
    P, O = prob
    comm, lps, Ks = _setup(dda, P, nparts)
    Fs = [torch.from_numpy(lp.F).cuda() for lp in lps]
    ds, it, rr, st = comm.pcg_solve(Fs, tol=1e-10, precond="bj")
    assert st == dda.OK and rr <= 1.01e-10
    do, ito, rro, sto = O.pcg(P.F, tol=1e-10, precond="bj")
    assert abs(it - ito) <= max(2, int(0.01 * ito))
    dm, _, _, _ = O.pcg(P.F, tol=1e-300, maxit=it, precond="bj")
    d = np.concatenate([t.cpu().numpy() for t in ds])
    assert np.linalg.norm(d - dm) / np.linalg.norm(dm) <= 1e-9


def test_pcg_dist_warm_and_zero(dda, prob, dist_version):
    P, O = prob
    comm, lps, Ks = _setup(dda, P, 3)
    Fs = [torch.from_numpy(lp.F).cuda() for lp in lps]
    ds, it, rr, st = comm.pcg_solve(Fs)
    d0s = [d.clone() for d in ds]
    _, it2, rr2, st2 = comm.pcg_solve(Fs, d0s=d0s)
    assert st2 == dda.OK and it2 <= 1
    zs, itz, rrz, stz = comm.pcg_solve([torch.zeros_like(F) for F in Fs])
    assert stz == dda.OK and itz == 0 and all(not z.any() for z in zs)
    # iteration cap not a multiple of the host-check chunk (device-side loop state, v2)
    _, it5, rr5, st5 = comm.pcg_solve(Fs, maxit=13)
    assert st5 == dda.ERR_NO_CONVERGENCE and it5 == 13 and rr5 > 1e-10


def test_pcg_dist_nccl_single_rank(dda, prob, dist_version):
    P, O = prob
    uid = dda.Comm.unique_id()
    comm = dda.Comm.nccl(1, 0, uid)
    b = row_bounds(P.n, 1)
    lp = local_from_slope(P, b, 0)
    K = dda.build_local(lp)
    comm.attach(0, K, lp)
    ds, it, rr, st = comm.pcg_solve([torch.from_numpy(lp.F).cuda()])
    Kg = dda.build_from_problem(P)
    d2, it2, rr2, st2 = Kg.pcg_solve(torch.from_numpy(P.F).cuda())
    assert st == st2 == dda.OK and abs(it - it2) <= 1
    assert torch.linalg.norm(ds[0] - d2) / torch.linalg.norm(d2) <= 1e-9
