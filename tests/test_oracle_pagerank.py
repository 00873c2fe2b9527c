"""Pins for the PageRank oracle (Alg. 1 l.26-29; readings R5-R7).

* a dense Google-matrix power iteration (matrix form, not the push loop) on n <= 12,
* networkx.pagerank (its own implementation) converged, vs the oracle run to convergence,
* closed forms: directed cycle / complete digraph / edgeless graph stay exactly uniform;
  the two-node graph a->b converges to (1/(2+d*... )) = (0.350877..., 0.649122...),
* the ranks sum to 1.
"""
import networkx as nx
import numpy as np
import pytest

import oracle
import sagegen as sg


def google_power(g, d, iters):
    n = g.n
    P = np.zeros((n, n))
    for u in range(n):
        deg = g.off[u + 1] - g.off[u]
        if deg == 0:
            P[u, :] = 1.0 / n          # dangling mass spread uniformly (R5)
        else:
            P[u, g.col[g.off[u]:g.off[u + 1]]] = 1.0 / deg
    G = d * P + (1 - d) / n
    x = np.full(n, 1.0 / n)
    for _ in range(iters):
        x = x @ G
    return x


@pytest.mark.parametrize("seed", range(30))
def test_dense_google_matrix(seed):
    n = 2 + seed % 11
    g = sg.random_graph(n, 2 * n, 300 + seed, symmetric=bool(seed % 2))
    for iters in (0, 1, 20):
        x = oracle.pagerank(g.off, g.col, 0.85, iters)
        assert np.max(np.abs(x - google_power(g, 0.85, iters)) / google_power(g, 0.85, iters)) < 1e-13


def test_networkx_converged():
    g = sg.rmat(10, 8, seed=5, symmetric=False)
    G = nx.DiGraph()
    G.add_nodes_from(range(g.n))
    src = np.repeat(np.arange(g.n), np.diff(g.off))
    G.add_edges_from(zip(src.tolist(), g.col.tolist()))
    ref = nx.pagerank(G, alpha=0.85, tol=1e-15, max_iter=1000)
    ref = np.array([ref[v] for v in range(g.n)])
    x = oracle.pagerank(g.off, g.col, 0.85, 300)
    assert np.max(np.abs(x - ref) / ref) < 1e-9


@pytest.mark.parametrize("kind", ["cycle", "complete", "edgeless"])
def test_uniform_closed_forms(kind):
    n = 7
    if kind == "cycle":
        e = [(i, (i + 1) % n) for i in range(n)]
    elif kind == "complete":
        e = [(i, j) for i in range(n) for j in range(n) if i != j]
    else:
        e = []
    g = sg.from_edges(n, e)
    for iters in (1, 5, 20):
        x = oracle.pagerank(g.off, g.col, 0.85, iters)
        assert np.allclose(x, 1.0 / n, rtol=1e-14, atol=0)


def test_two_node_closed_form():
    # a -> b, b dangling: stationary x_a = (1-d)/2 + d*x_b/2, x_b = (1-d)/2 + d*(x_a + x_b/2)
    # => x_a = 1/(2+d) ... with d = 0.85: x_a = 0.5/1.425 = 0.3508771929824561
    g = sg.from_edges(2, [(0, 1)])
    x = oracle.pagerank(g.off, g.col, 0.85, 200)
    assert abs(x[0] - 0.5 / 1.425) < 1e-15 and abs(x[1] - (1 - 0.5 / 1.425)) < 1e-15


def test_sums_to_one():
    g = sg.rmat(12, 16, seed=1, symmetric=False)
    x = oracle.pagerank(g.off, g.col, 0.85, 20)
    assert abs(x.sum() - 1.0) < 1e-12
    assert np.all(x >= 0.15 / g.n * (1 - 1e-12))


def test_pagerank_step_composes_to_pagerank():
    """pagerank_step applied K times from x0 = 1/N reproduces pagerank(K) bit for bit (same
    arithmetic in the same order), and a hand-computed step on a 3-vertex graph."""
    g = sg.rmat(9, 8, seed=4, symmetric=False)
    x = np.full(g.n, 1.0 / g.n)
    for _ in range(7):
        x = oracle.pagerank_step(g.off, g.col, x, 0.85)
    assert np.array_equal(x, oracle.pagerank(g.off, g.col, 0.85, 7))
    h = sg.from_edges(3, [(0, 1), (0, 2), (1, 2)], False, "tri")     # vertex 2 dangles
    x0 = np.array([0.5, 0.3, 0.2])
    d = 0.85
    exp = np.array([0.0, 0.5 / 2, 0.5 / 2 + 0.3]) * d + (1 - d) / 3 + d * 0.2 / 3
    assert np.allclose(oracle.pagerank_step(h.off, h.col, x0, d), exp, rtol=0, atol=1e-15)
