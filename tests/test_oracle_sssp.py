"""Pins for the SSSP oracle (reading R4).

* brute-force Bellman-Ford (n-1 full relaxation sweeps, exact uint64) on tiny graphs,
* scipy.sparse.csgraph.dijkstra (float64 is exact for integer sums < 2^53),
* w == 1 reduces to the BFS levels (c1),
* the SSSP certificate accepts the oracle's answer and rejects perturbations,
* a path whose length exceeds UINT32_MAX is reported as overflow.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import dijkstra

import oracle
import sagegen as sg

U32MAX = np.iinfo(np.uint32).max


def bellman_ford(g, w, s):
    INF = None
    d = [INF] * g.n
    d[s] = 0
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    for _ in range(g.n):
        for k in range(g.m):
            u, v = int(src[k]), int(g.col[k])
            if d[u] is not None and (d[v] is None or d[u] + int(w[k]) < d[v]):
                d[v] = d[u] + int(w[k])
    return d


@pytest.mark.parametrize("seed", range(40))
def test_tiny_vs_bellman_ford(seed):
    n = 3 + seed % 10
    g = sg.random_graph(n, 3 * n, 500 + seed, symmetric=bool(seed % 2))
    w = sg.weights(g, seed, wmax=9 if seed % 3 else 255)
    for s in range(n):
        dist, ovf = oracle.sssp(g.off, g.col, w, s)
        assert not ovf
        ref = bellman_ford(g, w, s)
        exp = np.array([U32MAX if x is None else x for x in ref], dtype=np.uint32)
        assert np.array_equal(dist, exp), (seed, s)
        assert oracle.check_sssp(g.off, g.col, w, s, dist) == 0


@pytest.mark.parametrize("sym", [True, False])
def test_scipy_dijkstra(sym):
    g = sg.rmat(13, 8, seed=4, symmetric=sym)
    w = sg.weights(g, 7)
    A = sp.csr_matrix((w.astype(np.float64), g.col, g.off), shape=(g.n, g.n))
    srcs = sg.sources(g, 3, seed=9)
    D = dijkstra(A, indices=srcs)
    for i, s in enumerate(srcs):
        dist, _ = oracle.sssp(g.off, g.col, w, int(s))
        exp = np.where(np.isinf(D[i]), U32MAX, D[i]).astype(np.uint64)
        assert np.array_equal(dist.astype(np.uint64), exp)


def test_unit_weights_equal_bfs():
    g = sg.rmat(12, 16, seed=2, symmetric=True)
    w = np.ones(g.m, dtype=np.uint32)
    for s in sg.sources(g, 3):
        dist, _ = oracle.sssp(g.off, g.col, w, int(s))
        lev = oracle.bfs(g.off, g.col, int(s))
        exp = np.where(lev < 0, U32MAX, lev).astype(np.uint32)
        assert np.array_equal(dist, exp)


def test_certificate_rejects_perturbations():
    total = rejected = 0
    for seed in range(25):
        n = 4 + seed % 7
        g = sg.random_graph(n, 3 * n, 900 + seed, symmetric=bool(seed % 2))
        w = sg.weights(g, seed, wmax=5)
        s = seed % n
        dist, _ = oracle.sssp(g.off, g.col, w, s)
        for v in range(n):
            for delta in (-1, 1, 3):
                bad = dist.astype(np.int64).copy()
                if bad[v] == U32MAX:
                    bad[v] = 7
                else:
                    bad[v] = max(0, bad[v] + delta)
                bad = bad.astype(np.uint32)
                if np.array_equal(bad, dist):
                    continue
                total += 1
                rejected += oracle.check_sssp(g.off, g.col, w, s, bad) != 0
    assert total > 200 and rejected == total


def test_overflow_detected():
    g = sg.from_edges(4, [(0, 1), (1, 2), (2, 3)])
    w = np.array([U32MAX - 5, 3, 10], dtype=np.uint32)
    dist, ovf = oracle.sssp(g.off, g.col, w, 0)
    assert ovf
    assert dist[1] == U32MAX - 5 and dist[2] == U32MAX - 2
    w = np.array([U32MAX - 5, 3, 1], dtype=np.uint32)   # reaches exactly U32MAX-1
    dist, ovf = oracle.sssp(g.off, g.col, w, 0)
    assert not ovf and dist[3] == U32MAX - 1
