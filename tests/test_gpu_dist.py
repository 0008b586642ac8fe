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
from partition_ref import row_bounds, local_from_slope
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


@pytest.fixture(params=["v7", "v6", "v5", "v4", "v4_seq", "v3", "v2"])
def dist_version(request, monkeypatch):
    """v7 = one persistent cooperative kernel PER partition, the launches running concurrently and
    meeting only through published rank totals and an arrival counter (DDA_DIST_VERSION=7, the
    one-process-per-GPU structure under loopback); v6 = every partition in one persistent cooperative kernel, halo rows read from their owners'
    r~ / p_old and every sum a fixed-order read of all partitions' partials (loopback default; NCCL runs
    v4); v5 = the v4 iteration with the halo read from the owners' rows (peer loads) and the allreduce
    taken inside phase B (DDA_DIST_VERSION=5); v4 = one halo copy and one allreduce per iteration
    (DDA_DIST_VERSION=4; the NCCL transport always runs it), phase A of the interior rows overlapped with
    the halo on a second stream; v4_seq = the same without the overlap (DDA_DIST_OVERLAP=0); v3 = two
    halos and three allreduces (DDA_DIST_VERSION=3); v2 = the unscaled loop (DDA_DIST_SCALED=0).  Read on
    every solve."""
    monkeypatch.delenv("DDA_DIST_SCALED", raising=False)
    monkeypatch.delenv("DDA_DIST_VERSION", raising=False)
    monkeypatch.delenv("DDA_DIST_OVERLAP", raising=False)
    if request.param == "v2":
        monkeypatch.setenv("DDA_DIST_SCALED", "0")
    elif request.param in ("v3", "v4", "v4_seq", "v5", "v7"):
        monkeypatch.setenv("DDA_DIST_VERSION", request.param[1])
        if request.param == "v4_seq":
            monkeypatch.setenv("DDA_DIST_OVERLAP", "0")
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


def _setup_device(dda, P, nparts, shuffle_springs=False):
    """Partitions built behind the C ABI (dda_build_matrix_dist) from the GLOBAL spring list."""
    b = dda.row_bounds(P.n, nparts)
    comm = dda.Comm.loopback(nparts)
    t = dda.problem_to_device(P)
    Ks, Fs = [], []
    for r in range(nparts):
        r0, r1 = int(b[r]), int(b[r + 1])
        Ks.append(comm.build_matrix_dist(r, P.n, b, t["kdiag"][r0:r1].contiguous(), t["bi"], t["bj"], t["pen"],
                                         t["e"], t["g"]))
        Fs.append(t["F"][6 * r0:6 * r1].contiguous())
    return comm, b, Ks, Fs


@pytest.mark.parametrize("nparts", [1, 2, 3, 4])
def test_build_matrix_dist_matches_host_reference(dda, prob, nparts):
    """The device partition (selection, halo, numbering, assembly, plan) equals the host reference
    tests/partition_ref.py: local structure and values bit-exact against the ORACLE's assembly of the
    reference local problem, and the same n_halo / send / receive plan."""
    P, O = prob
    comm, b, Ks, Fs = _setup_device(dda, P, nparts)
    bref = row_bounds(P.n, nparts)
    assert np.array_equal(b, bref)
    for r in range(nparts):
        lp = local_from_slope(P, bref, r)
        Ol = oracle.OracleMatrix(lp.n_local, lp.kdiag, lp.bi, lp.bj, lp.pen, lp.e, lp.g)
        S, ex = Ol.export(), Ks[r].export()
        for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
            assert np.array_equal(ex[k], getattr(S, k)), (r, k)
        assert np.array_equal(ex["diag"], S.diag) and np.array_equal(ex["upper"], S.upper), r
        inf = comm.info(r)
        assert inf["n_own"] == lp.n_own and inf["n_halo"] == lp.n_halo
        assert np.array_equal(inf["send_counts"], lp.send_counts)
        assert np.array_equal(inf["recv_counts"], lp.recv_counts)
        assert np.array_equal(inf["send_idx"], lp.send_idx)


@pytest.mark.parametrize("nparts", [2, 4])
def test_pcg_dist_device_built(dda, prob, nparts, dist_version):
    """Partitions from dda_build_matrix_dist solved by dda_pcg_solve_dist, vs the oracle (Z17)."""
    P, O = prob
    comm, b, Ks, Fs = _setup_device(dda, P, nparts)
    ds, it, rr, st = comm.pcg_solve(Fs, tol=1e-10, precond="bj")
    assert st == dda.OK and rr <= 1.01e-10
    do, ito, rro, sto = O.pcg(P.F, tol=1e-10, precond="bj")
    assert abs(it - ito) <= max(2, int(0.01 * ito))
    dm, _, _, _ = O.pcg(P.F, tol=1e-300, maxit=it, precond="bj")
    d = np.concatenate([t.cpu().numpy() for t in ds])
    assert np.linalg.norm(d - dm) / np.linalg.norm(dm) <= 1e-9
    y = np.concatenate([t.cpu().numpy() for t in comm.spmv([torch.from_numpy(d[6 * b[r]:6 * b[r + 1]].copy()).cuda()
                                                               for r in range(nparts)])])
    assert np.linalg.norm(y - O.spmv(d)) <= 1e-12 * np.linalg.norm(y)


def test_build_matrix_dist_errors(dda, prob):
    P, O = prob
    comm = dda.Comm.loopback(2)
    t = dda.problem_to_device(P)
    b = dda.row_bounds(P.n, 2)
    kd = t["kdiag"][: int(b[1])].contiguous()
    for bad_b in (np.array([0, 5, 5], np.int32), np.array([1, 5, P.n], np.int32)):
        kdb = t["kdiag"][: int(bad_b[1] - bad_b[0])].contiguous()
        with pytest.raises(dda.DDAError):
            comm.build_matrix_dist(0, P.n, bad_b, kdb, t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    with pytest.raises(dda.DDAError):                 # partition index out of range
        comm.build_matrix_dist(2, P.n, b, kd, t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    bi = t["bi"].clone()
    bi[3] = P.n                                       # id out of range
    with pytest.raises(dda.DDAError):
        comm.build_matrix_dist(0, P.n, b, kd, bi, t["bj"], t["pen"], t["e"], t["g"])


def test_pcg_dist_nccl_single_rank_oracle(dda, prob):
    """NCCL transport (one rank), partition built on the device, against the oracle (Z17)."""
    P, O = prob
    comm = dda.Comm.nccl(1, 0, dda.Comm.unique_id())
    t = dda.problem_to_device(P)
    b = dda.row_bounds(P.n, 1)
    comm.build_matrix_dist(0, P.n, b, t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
    ds, it, rr, st = comm.pcg_solve([t["F"]])
    assert st == dda.OK and rr <= 1.01e-10
    do, ito, _, _ = O.pcg(P.F, tol=1e-10, precond="bj")
    assert abs(it - ito) <= max(2, int(0.01 * ito))
    dm, _, _, _ = O.pcg(P.F, tol=1e-300, maxit=it, precond="bj")
    assert np.linalg.norm(ds[0].cpu().numpy() - dm) / np.linalg.norm(dm) <= 1e-9
    comm.free()


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
