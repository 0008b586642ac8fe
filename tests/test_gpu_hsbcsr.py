"""NEXT-2 ablation on the GPU: the paper's HSBCSR two-stage SpMV (dda_hsbcsr_*) against
the oracle through the C ABI: the half-slice layout of d-data / nd-data-up exactly as P:184 (Fig. 6)
describes it (rebuilt here from the oracle's blocks), and y = K x componentwise <= 1e-12, on the
tiny slope, a ragged 1k slope and the case-1-sized matrix (4361 + 18731 blocks)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from synth import case1_like, make_slope, preset, random_vector

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (no CPU fallback exists)")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


def _problem(name):
    if name == "case1":
        return case1_like()
    P = make_slope(preset("tiny") if name == "tiny" else preset(1000, seed=1041))
    return P.n, P.kdiag, P.bi, P.bj, P.pen, P.e, P.g, P.F


@pytest.mark.parametrize("name", ["tiny", "ragged_1k", "case1"])
def test_hsbcsr_layout_and_spmv(dda, name):
    n, kd, bi, bj, pen, e, g, F = _problem(name)
    O = oracle.OracleMatrix(n, kd, bi, bj, pen, e, g)
    S = O.export()
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    K = dda.build_matrix(dev(kd), dev(bi), dev(bj), dev(pen), dev(e), dev(g))
    H = dda.HSBCSR(K)
    dd, nd = H.export()
    for arr, blocks in ((dd, S.diag), (nd, S.upper)):
        nb = blocks.shape[0]
        stride = ((6 * nb + 31) // 32) * 32
        assert arr.shape == (6, stride)                                  # slices padded to 32 doubles
        want = np.zeros((6, stride))
        want[:, :6 * nb] = np.transpose(blocks, (1, 0, 2)).reshape(6, 6 * nb)   # slice r = row r of every block
        assert np.array_equal(arr, want)
    x = random_vector(n, 17)
    y = H.spmv(dev(x)).cpu().numpy()
    yo = O.spmv(x)
    ip, ix, dv = O.full_csr()
    bound = np.zeros(6 * n)
    np.add.at(bound, np.repeat(np.arange(6 * n), np.diff(ip)), np.abs(dv) * np.abs(x[ix]))
    assert (np.abs(y - yo) <= 1e-12 * bound).all()
    assert np.array_equal(y, H.spmv(dev(x)).cpu().numpy())             # deterministic (no atomics)
    if name == "case1":
        assert n == 4361 and K.nnzb == 18731
