"""The library's caching device allocator (csrc/alloc.cu, include/dda.h dda_memory_*):
a rebuild of the same system after dda_matrix_free reuses the cached blocks, results are
unchanged by reuse, and dda_memory_release empties the cache."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from synth import make_slope, preset

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as m
    return m


def test_rebuild_reuses_cached_blocks(dda):
    P = make_slope(preset(20000, seed=1043))
    t = dda.problem_to_device(P)
    dda.memory_release()
    assert dda.memory_cached() == 0
    sols = []
    cached = []
    for _ in range(3):
        K = dda.build_matrix(t["kdiag"], t["bi"], t["bj"], t["pen"], t["e"], t["g"])
        d, it, rr, st = K.pcg_solve(t["F"])
        assert st == dda.OK and rr <= 1.01e-10
        sols.append(d.cpu().numpy())
        during = dda.memory_cached()
        K.free()
        cached.append((during, dda.memory_cached()))
    # after the first free the cache holds the matrix; later builds take it back (cache shrinks
    # while the matrix is alive) and return it on free
    assert cached[0][1] > 0
    assert cached[1][0] < cached[0][1] and cached[2][0] < cached[1][1]
    assert cached[2][1] == cached[1][1]
    assert np.array_equal(sols[0], sols[1]) and np.array_equal(sols[1], sols[2])
    dda.memory_release()
    assert dda.memory_cached() == 0
