"""GPU parity on adversarial structures the slope generator never produces:
rows with many blocks (> 9: the second pass of the 9-entry block list in the
warp row routine), a hub block touching every other block, random sparse
graphs, n = 1 and two blocks.  Inputs are random SPD systems assembled from
springs with SPD diagonal terms; the oracle is the reference."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


def random_system(n, pairs, seed, diag_scale=20.0):
    rng = np.random.default_rng(seed)
    kd = rng.standard_normal((n, 6, 6))
    kd = np.einsum("bij,bkj->bik", kd, kd) + diag_scale * np.eye(6)
    pairs = np.asarray(pairs, np.int64).reshape(-1, 2)
    flip = rng.random(len(pairs)) < 0.5
    bi = np.where(flip, pairs[:, 1], pairs[:, 0]).astype(np.int32)
    bj = np.where(flip, pairs[:, 0], pairs[:, 1]).astype(np.int32)
    m = len(bi)
    pen = rng.uniform(0.5, 2.0, m)
    e = rng.standard_normal((m, 6))
    g = rng.standard_normal((m, 6))
    F = rng.standard_normal(6 * n)
    return kd, bi, bj, pen, e, g, F


def check(dda, n, pairs, seed, pcs=("bj", "ssor_ai", "ilu0")):
    kd, bi, bj, pen, e, g, F = random_system(n, pairs, seed)
    O = oracle.OracleMatrix(n, kd, bi, bj, pen, e, g)
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    K = dda.build_matrix(dev(kd), dev(bi), dev(bj), dev(pen), dev(e), dev(g))
    S, ex = O.export(), K.export()
    for k in ("row_ptr", "col_idx", "low_ptr", "low_row", "low_to_up"):
        assert np.array_equal(ex[k], getattr(S, k)), k
    assert np.array_equal(ex["diag"], S.diag) and np.array_equal(ex["upper"], S.upper)
    x = np.random.default_rng(seed + 1).uniform(-1, 1, 6 * n)
    y = K.spmv(dev(x)).cpu().numpy()
    yf = K.spmv_full(dev(x)).cpu().numpy()
    yo = O.spmv(x)
    ip, ix, dv = O.full_csr()
    bound = np.zeros(6 * n)
    np.add.at(bound, np.repeat(np.arange(6 * n), np.diff(ip)), np.abs(dv) * np.abs(x[ix]))
    assert (np.abs(y - yo) <= 1e-12 * bound).all()
    assert (np.abs(yf - yo) <= 1e-12 * bound).all()
    for pc in pcs:
        d, it, rr, st = K.pcg_solve(dev(F), tol=1e-10, precond=pc)
        assert st == dda.OK and rr <= 1.01e-10, (pc, st, rr)
        do, ito, rro, sto = O.pcg(F, tol=1e-10, precond=pc)
        assert abs(it - ito) <= max(2, int(0.02 * ito)), (pc, it, ito)
        dm, _, _, _ = O.pcg(F, tol=1e-300, maxit=it, precond=pc)
        assert np.linalg.norm(d.cpu().numpy() - dm) <= 1e-9 * np.linalg.norm(dm), pc


def test_hub_block(dda):
    n = 41                                   # block 0 touches all 40 others: row 0 has 40 upper blocks,
    pairs = [(0, j) for j in range(1, n)]    # every other row has block 0 as a lower entry
    pairs += [(j, j + 1) for j in range(1, n - 1)]
    check(dda, n, pairs, 1)


def test_hub_in_the_middle(dda):
    n = 60
    hub = 30                                 # 30 lower + 29 upper blocks in one row
    pairs = [(min(hub, j), max(hub, j)) for j in range(n) if j != hub]
    check(dda, n, pairs, 2)


@pytest.mark.parametrize("seed", [3, 4])
def test_random_graph(dda, seed):
    rng = np.random.default_rng(seed)
    n = 300
    a = rng.integers(0, n, 3000); b = rng.integers(0, n, 3000)
    keep = a != b
    pairs = np.stack([a[keep], b[keep]], 1)  # duplicates kept: several springs per block pair
    check(dda, n, pairs, seed)


def test_single_block(dda):
    n = 1
    kd, bi, bj, pen, e, g, F = random_system(1, np.zeros((0, 2)), 5)
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    K = dda.build_matrix(dev(kd), dev(bi), dev(bj), dev(pen), dev(e.reshape(0, 6)), dev(g.reshape(0, 6)))
    assert K.n == 1 and K.nnzb == 0
    d, it, rr, st = K.pcg_solve(dev(F), precond="bj")
    assert st == dda.OK and it == 1
    assert np.allclose(kd[0] @ d.cpu().numpy(), F, rtol=1e-12, atol=1e-12)


def test_two_blocks(dda):
    check(dda, 2, [(0, 1), (1, 0), (0, 1)], 6)
