"""Input generators (test infrastructure): deterministic, well-formed CSR, seeded sources/weights."""
import numpy as np

import sagegen as sg


def test_rmat_deterministic_and_clean():
    a = sg.rmat(12, 16, seed=1)
    b = sg.rmat(12, 16, seed=1)
    assert np.array_equal(a.off, b.off) and np.array_equal(a.col, b.col)
    c = sg.rmat(12, 16, seed=2)
    assert not (len(c.col) == len(a.col) and np.array_equal(c.col, a.col))
    src = np.repeat(np.arange(a.n), np.diff(a.off))
    assert np.all(src != a.col)                                   # no self loops
    for u in range(a.n):
        r = a.col[a.off[u]:a.off[u + 1]]
        assert np.all(np.diff(r) > 0)                             # sorted, no duplicates
    fwd = set(zip(src.tolist(), a.col.tolist()))
    assert all((v, u) in fwd for (u, v) in fwd)                   # symmetric


def test_rmat16_shape_matches_survey():
    g = sg.rmat(16, 16, seed=1)
    # SURVEY Appendix A (scratch, seed 1): ~1.82e6 arcs, 28.7% isolated, max degree ~9.7e3
    assert 1.78e6 < g.m < 1.86e6
    assert 0.27 < np.mean(np.diff(g.off) == 0) < 0.30
    assert 8e3 < np.diff(g.off).max() < 1.2e4


def test_weights_symmetric_and_in_range():
    g = sg.rmat(10, 8, seed=3)
    w = sg.weights(g, 5)
    assert w.min() >= 1 and w.max() <= 255
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    d = {(int(u), int(v)): int(x) for u, v, x in zip(src, g.col, w)}
    assert all(d[(v, u)] == x for (u, v), x in d.items())


def test_sources_have_out_arcs():
    g = sg.rmat(10, 4, seed=3)
    s = sg.sources(g, 64, seed=2)
    assert np.all(np.diff(g.off)[s] > 0)
    assert np.array_equal(s, sg.sources(g, 64, seed=2))


def test_small_twitter_and_uk_like():
    t = sg.twitter_like(n=20000, tuples=400000, seed=1, cmin=8, cmax=2048)
    assert t.m > 300000 and np.diff(t.off).max() > 2000
    u = sg.uk_like(n=50000, seed=1, n_tendrils=20, tmin=50, tmax=100, hmax=4096)
    assert u.m > 10 * u.n // 2
