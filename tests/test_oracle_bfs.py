"""Pins for the BFS oracle (Alg. 1 l.1-6).

The oracle's FIFO BFS is checked against things that do not share its algorithm:
* boolean adjacency-matrix powers (hop distance = first k with (A^k)[s, v] > 0),
* scipy.sparse.csgraph.shortest_path(unweighted=True),
* the level certificate, which must reject every single-entry perturbation,
* the symmetric-graph invariant |level(u) - level(v)| <= 1 (north_star).
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import shortest_path

import oracle
import sagegen as sg


def brute_levels(g, s):
    n = g.n
    A = np.zeros((n, n), dtype=bool)
    for u in range(n):
        A[u, g.col[g.off[u]:g.off[u + 1]]] = True
    lev = np.full(n, -1, dtype=np.int32)
    reach = np.zeros(n, dtype=bool)
    reach[s] = True
    lev[s] = 0
    cur = reach.copy()
    for k in range(1, n + 1):
        cur = (cur.astype(np.int64) @ A.astype(np.int64)) > 0   # vertices at walk length k
        new = cur & ~reach
        lev[new] = k
        reach |= cur
    return lev


HAND = {
    "path": (5, [(0, 1), (1, 2), (2, 3), (3, 4)], False),
    "star": (6, [(0, i) for i in range(1, 6)], True),
    "cycle": (5, [(i, (i + 1) % 5) for i in range(5)], False),
    "complete": (5, [(i, j) for i in range(5) for j in range(5) if i != j], False),
    "selfloop_dup": (4, [(0, 0), (0, 1), (0, 1), (1, 2), (2, 2), (2, 3)], False),
    "isolated_src": (4, [(1, 2), (2, 3)], True),
    "single": (1, [], False),
    "disconnected": (6, [(0, 1), (1, 0), (3, 4), (4, 5)], True),
}


@pytest.mark.parametrize("name", sorted(HAND))
def test_hand_graphs_vs_brute_force(name):
    n, edges, sym = HAND[name]
    g = sg.from_edges(n, edges, symmetric=sym)
    for s in range(n):
        lev = oracle.bfs(g.off, g.col, s)
        assert np.array_equal(lev, brute_levels(g, s)), (name, s)
        assert oracle.check_bfs(g.off, g.col, s, lev) == 0


def test_hand_values():
    g = sg.from_edges(5, HAND["path"][1])
    assert oracle.bfs(g.off, g.col, 0).tolist() == [0, 1, 2, 3, 4]
    assert oracle.bfs(g.off, g.col, 2).tolist() == [-1, -1, 0, 1, 2]
    g = sg.from_edges(4, HAND["isolated_src"][1], symmetric=True)
    assert oracle.bfs(g.off, g.col, 0).tolist() == [0, -1, -1, -1]


@pytest.mark.parametrize("seed", range(40))
def test_random_tiny_vs_brute_force(seed):
    n = 3 + seed % 10
    g = sg.random_graph(n, 2 * n, seed, symmetric=bool(seed % 2))
    for s in range(n):
        assert np.array_equal(oracle.bfs(g.off, g.col, s), brute_levels(g, s))


@pytest.mark.parametrize("sym", [True, False])
def test_scipy_rmat(sym):
    g = sg.rmat(13, 8, seed=3, symmetric=sym)
    A = sp.csr_matrix((np.ones(g.m), g.col, g.off), shape=(g.n, g.n))
    srcs = sg.sources(g, 4, seed=5)
    D = shortest_path(A, unweighted=True, indices=srcs)
    for i, s in enumerate(srcs):
        lev = oracle.bfs(g.off, g.col, int(s))
        exp = np.where(np.isinf(D[i]), -1, D[i]).astype(np.int32)
        assert np.array_equal(lev, exp)


def test_symmetric_invariant_and_certificate():
    g = sg.rmat(12, 16, seed=1, symmetric=True)
    s = int(sg.sources(g, 1)[0])
    lev = oracle.bfs(g.off, g.col, s)
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    both = (lev[src] >= 0) & (lev[g.col] >= 0)
    assert np.all(np.abs(lev[src][both] - lev[g.col][both]) <= 1)
    # reached set is closed under arcs
    assert np.all(lev[g.col][lev[src] >= 0] >= 0)
    assert oracle.check_bfs(g.off, g.col, s, lev) == 0


def test_certificate_rejects_perturbations():
    rng = np.random.default_rng(0)
    rejected = 0
    total = 0
    for seed in range(30):
        n = 4 + seed % 7
        g = sg.random_graph(n, 2 * n, 100 + seed, symmetric=bool(seed % 2))
        s = int(seed % n)
        lev = oracle.bfs(g.off, g.col, s)
        for v in range(n):
            for delta in (-2, -1, 1, 2):
                bad = lev.copy()
                bad[v] = max(-1, bad[v] + delta)
                if np.array_equal(bad, lev):
                    continue
                total += 1
                rejected += oracle.check_bfs(g.off, g.col, s, bad) != 0
    assert total > 300 and rejected == total
