"""Pins of the online Sampling-based Reordering oracle (NEXT #3; §6; reading R19b).

The weighted sample is pinned to the offline sample (weights 1 == sample_tiles), to scaling (all
weights k: every stage count scales by k, so the round's permutation is unchanged — a dropped or
doubled occurrence changes it), to exclusion (weight 0 rows contribute nothing: a round whose
sample is one vertex's rows equals the round on the graph with every other row emptied), and the
BFS-driven driver to its definition on a hand-checkable case.
"""
import numpy as np

import oracle
import sagegen as sg


def test_weighted_sample_equals_offline_sample():
    g = sg.rmat(9, 8, seed=2, symmetric=True)
    tp, mem = oracle.sample_tiles(g.off, g.col, 16, 4, 4)
    tw, mw = oracle.sample_tiles_weighted(g.off, g.col, np.ones(g.n, dtype=np.int64), 16, 4, 4)
    assert np.array_equal(tp, tw) and np.array_equal(mem, mw)


def test_uniform_weight_scaling_keeps_the_round():
    g = sg.rmat(9, 8, seed=3, symmetric=True)
    r1 = oracle.reorder_round_weighted(g.off, g.col, None, np.ones(g.n, dtype=np.int64), 16, 4, 4, 8)
    r3 = oracle.reorder_round_weighted(g.off, g.col, None, np.full(g.n, 3, dtype=np.int64), 16, 4, 4, 8)
    assert r1[4] > 0 and r1[5] > 0
    assert np.array_equal(r1[3], r3[3]) and np.array_equal(r1[1], r3[1])
    # and it is the offline round
    off2, col2, _, sig, _ = oracle.reorder(g.off, g.col, None, rounds=1, B=16, M=4, A=4, S=8)
    assert np.array_equal(sig, r1[3]) and np.array_equal(col2, r1[1])


def test_zero_weight_rows_are_not_sampled():
    g = sg.rmat(8, 8, seed=4, symmetric=False)
    wts = np.zeros(g.n, dtype=np.int64)
    keep = np.nonzero(np.diff(g.off) >= 8)[0][:20]
    wts[keep] = 1
    rw = oracle.reorder_round_weighted(g.off, g.col, None, wts, 8, 4, 0, 4)
    # the same sample built from a CSR whose other rows are empty
    deg = np.zeros(g.n, dtype=np.int64)
    deg[keep] = np.diff(g.off)[keep]
    off_k = np.zeros(g.n + 1, dtype=np.int64)
    np.cumsum(deg, out=off_k[1:])
    col_k = np.concatenate([g.col[g.off[u]:g.off[u + 1]] for u in range(g.n) if deg[u]])
    tp, mem = oracle.sample_tiles(off_k, col_k, 8, 4, 0)
    st = oracle.reorder_stages(g.n, tp, mem, 4)
    if st["mover"].sum():
        sig, _ = oracle.reorder_match(g.n, 4, st)
        assert np.array_equal(sig, rw[3])
    else:
        assert np.array_equal(rw[3], np.arange(g.n))


def test_online_driver_thresholds_and_answers():
    g = sg.rmat(10, 8, seed=5, symmetric=True)
    srcs = [int(s) for s in sg.sources(g, 6, seed=2)]
    # threshold above any single query's sample: rounds happen every few queries
    sig, rounds, levels = oracle.online_reorder_bfs(g.off, g.col, srcs, threshold=3 * g.m, B=16, M=4, A=4)
    assert 1 <= rounds <= 3
    for s, lv in zip(srcs, levels):          # answers never change (original ids)
        assert np.array_equal(lv, oracle.bfs(g.off, g.col, s))
    assert np.array_equal(np.sort(sig), np.arange(g.n))
    # a huge threshold: no round, identity
    sig0, r0, _ = oracle.online_reorder_bfs(g.off, g.col, srcs, threshold=10 ** 12)
    assert r0 == 0 and np.array_equal(sig0, np.arange(g.n))
