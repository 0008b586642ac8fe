import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a); parity tests through the C ABI")
    config.addinivalue_line("markers", "slow: larger CPU cases (still a few seconds)")


@pytest.fixture(scope="session")
def tiny():
    from synth import make_slope, preset
    return make_slope(preset("tiny"))


@pytest.fixture(scope="session")
def tiny_oracle(tiny):
    import oracle
    return oracle.assemble(tiny)


@pytest.fixture(scope="session")
def paper():
    from synth import make_slope, preset
    return make_slope(preset("paper"))


def dense_from_springs(P):
    """Brute-force dense K (numpy, independent of the oracle): Kd (upper triangle
    mirrored, reading Z9) plus, per spring, the rank-1 term [e; g] p [e; g]^T
    placed on blocks (bi, bj) — P:104."""
    n = P.n
    K = np.zeros((6 * n, 6 * n))
    for i in range(n):
        U = np.triu(P.kdiag[i])
        K[6 * i:6 * i + 6, 6 * i:6 * i + 6] = U + np.triu(U, 1).T
    for s in range(P.m):
        w = np.concatenate([P.e[s], P.g[s]])
        idx = np.concatenate([6 * P.bi[s] + np.arange(6), 6 * P.bj[s] + np.arange(6)])
        K[np.ix_(idx, idx)] += P.pen[s] * np.outer(w, w)
    return K
