"""T0: the seeded input generator.  CPU only."""
import numpy as np

from synth import make_slope, preset, random_vector


def test_seed_determinism():
    a = make_slope(preset("tiny"))
    b = make_slope(preset("tiny"))
    for f in ("kdiag", "bi", "bj", "pen", "e", "g", "F"):
        assert np.array_equal(getattr(a, f), getattr(b, f)), f
    c = make_slope(preset("tiny", seed=77))
    assert not np.array_equal(a.e, c.e)


def test_shapes_and_ranges(tiny):
    P = tiny
    assert P.kdiag.shape == (P.n, 6, 6) and P.F.shape == (6 * P.n,)
    assert P.bi.dtype == np.int32 and P.bj.dtype == np.int32
    assert P.e.shape == (P.m, 6) and P.g.shape == (P.m, 6)
    assert (P.bi != P.bj).all() and P.bi.min() >= 0 and max(P.bi.max(), P.bj.max()) < P.n
    assert (P.pen > 0).all()
    # both orientations occur, so the stored-block transposition path is exercised (Z7)
    assert (P.bi < P.bj).any() and (P.bi > P.bj).any()


def test_contact_density_paper_scale(paper):
    # "~5 contacts/block" (BASELINE configs[1]); u = upper blocks per row ~ 3
    P = paper
    assert 9000 <= P.n <= 11000
    cpb = P.n_contacts / P.n
    assert 4.0 <= cpb <= 6.5, cpb
    pairs = np.unique(np.minimum(P.bi, P.bj).astype(np.int64) * P.n + np.maximum(P.bi, P.bj))
    u = pairs.size / P.n
    assert 2.5 <= u <= 3.5, u


def test_diagonal_terms_spd(tiny):
    ev = np.linalg.eigvalsh(tiny.kdiag)
    assert (ev > 0).all()
    assert np.array_equal(tiny.kdiag, np.transpose(tiny.kdiag, (0, 2, 1)))


def test_shuffle_is_a_relabelling():
    a = make_slope(preset("tiny"))
    b = make_slope(preset("tiny", shuffle=True))
    assert a.n == b.n and a.m == b.m
    # the multiset of diagonal terms is unchanged
    ka = np.sort(a.kdiag.reshape(a.n, -1), axis=0)
    kb = np.sort(b.kdiag.reshape(b.n, -1), axis=0)
    assert np.array_equal(ka, kb)


def test_random_vector():
    x = random_vector(10, 5)
    assert x.shape == (60,) and (np.abs(x) <= 1).all()
    assert np.array_equal(x, random_vector(10, 5))
