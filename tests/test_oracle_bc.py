"""Pins for the BC oracle (Alg. 1 l.8-24; Brandes' dependency accumulation).

* brute force: delta_s(v) = sum_t sigma_st(v) / sigma_st, with sigma counted by enumerating every
  shortest path of tiny graphs (n <= 9) — independent of the BFS/backward recursion;
* networkx.betweenness_centrality(normalized=False, endpoints=False) = sum over all sources
  (halved for undirected graphs);
* closed forms: the centre of a star of k leaves has BC k(k-1) over all sources (ordered pairs);
  the interior vertex i of a directed path 0->1->...->n-1 has delta_0(i) = n-1-i.
"""
import itertools

import networkx as nx
import numpy as np
import pytest

import oracle
import sagegen as sg


def _all_shortest_paths(adj, s, t):
    """Enumerate every shortest s-t path by BFS-layered DFS (brute force)."""
    n = len(adj)
    dist = {s: 0}
    frontier = [s]
    while frontier:
        nxt = []
        for u in frontier:
            for v in adj[u]:
                if v not in dist:
                    dist[v] = dist[u] + 1
                    nxt.append(v)
        frontier = nxt
    if t not in dist:
        return []
    paths = []

    def rec(path):
        u = path[-1]
        if u == t:
            paths.append(list(path))
            return
        for v in adj[u]:
            if dist.get(v) == dist[u] + 1 and dist[v] <= dist[t]:
                path.append(v)
                rec(path)
                path.pop()
    rec([s])
    return paths


def _brute_delta(g, s):
    adj = [list(g.col[g.off[u]:g.off[u + 1]]) for u in range(g.n)]
    d = np.zeros(g.n)
    for t in range(g.n):
        if t == s:
            continue
        ps = _all_shortest_paths(adj, s, t)
        if not ps:
            continue
        for v in range(g.n):
            if v in (s, t):
                continue
            d[v] += sum(1 for p in ps if v in p[1:-1]) / len(ps)
    return d


@pytest.mark.parametrize("seed", range(12))
def test_bc_brute_force_tiny(seed):
    g = sg.random_graph(9, 18, seed=seed, symmetric=bool(seed % 2))
    for s in range(g.n):
        got = oracle.bc(g.off, g.col, [s])
        exp = _brute_delta(g, s)
        exp[s] = 0.0
        assert np.allclose(got, exp, rtol=1e-12, atol=1e-12), (seed, s)


@pytest.mark.parametrize("sym", [True, False])
def test_bc_networkx(sym):
    g = sg.rmat(8, 8, seed=5, symmetric=sym)
    G = nx.Graph() if sym else nx.DiGraph()
    G.add_nodes_from(range(g.n))
    for u in range(g.n):
        for v in g.col[g.off[u]:g.off[u + 1]]:
            G.add_edge(u, int(v))
    ref = nx.betweenness_centrality(G, normalized=False)
    got = oracle.bc(g.off, g.col, np.arange(g.n))
    if sym:
        got = got / 2.0
    assert np.allclose(got, [ref[v] for v in range(g.n)], rtol=1e-9, atol=1e-9)


def test_bc_closed_forms():
    k = 7
    star = sg.from_edges(k + 1, [(0, i) for i in range(1, k + 1)], True, "star")
    bc = oracle.bc(star.off, star.col, np.arange(k + 1))
    assert bc[0] == k * (k - 1) and np.all(bc[1:] == 0)
    n = 10
    path = sg.from_edges(n, [(i, i + 1) for i in range(n - 1)], False, "path")
    d = oracle.bc(path.off, path.col, [0])
    assert np.array_equal(d, np.array([0.0] + [n - 1 - i for i in range(1, n)]))
