"""Oracle pins on CSRs that KEEP self-loops and duplicate arcs (reading R8: out(u) = stored arc
count; the ABI accepts such CSRs, so both sides must agree on them).  The CSRs are built by hand
here, not through sagegen (whose generators drop loops and duplicates).

* BFS: brute-force set-based frontier expansion,
* SSSP: brute-force Bellman-Ford over the arc list (duplicate arcs with different weights),
* PageRank: a dense power iteration with P[u, v] = multiplicity(u->v) / out(u),
* Sampling-based Reordering stage 1 (Fig. 5 reading R18): locality counted per member
  OCCURRENCE straight from the definition (a duplicate of v in its own tile is a mate).
"""
import numpy as np
import pytest

import oracle

ROWS = {0: [1, 1, 0, 2], 1: [2, 2], 2: [0, 3, 3, 3], 3: [], 4: [4, 4], 5: [5], 6: [0, 6, 6, 1, 1, 1]}
WTS = {0: [5, 2, 1, 9], 1: [3, 1], 2: [4, 7, 2, 6], 3: [], 4: [1, 1], 5: [3], 6: [2, 1, 1, 8, 1, 4]}


def multigraph(rows=ROWS, wts=WTS):
    n = max(rows) + 1
    off = np.zeros(n + 1, dtype=np.int64)
    for u in range(n):
        off[u + 1] = off[u] + len(rows.get(u, []))
    col = np.array([c for u in range(n) for c in rows.get(u, [])], dtype=np.int32)
    w = np.array([x for u in range(n) for x in wts.get(u, [])], dtype=np.uint32)
    return off, col, w


def brute_bfs(off, col, s):
    n = len(off) - 1
    lv = [-1] * n
    lv[s] = 0
    front, d = {s}, 0
    while front:
        nxt = set()
        for u in front:
            for v in col[off[u]:off[u + 1]]:
                if lv[v] < 0:
                    nxt.add(int(v))
        d += 1
        for v in nxt:
            lv[v] = d
        front = nxt
    return np.array(lv, dtype=np.int32)


def brute_sssp(off, col, w, s):
    n = len(off) - 1
    inf = 1 << 62
    d = [inf] * n
    d[s] = 0
    arcs = [(u, int(col[k]), int(w[k])) for u in range(n) for k in range(off[u], off[u + 1])]
    for _ in range(n):
        for u, v, x in arcs:
            if d[u] + x < d[v]:
                d[v] = d[u] + x
    return np.array([x if x < inf else 0xFFFFFFFF for x in d], dtype=np.uint32)


@pytest.mark.parametrize("s", range(7))
def test_bfs_sssp_on_multigraph(s):
    off, col, w = multigraph()
    assert np.array_equal(oracle.bfs(off, col, s), brute_bfs(off, col, s))
    d, ovf = oracle.sssp(off, col, w, s)
    assert not ovf and np.array_equal(d, brute_sssp(off, col, w, s))


@pytest.mark.parametrize("iters", [0, 1, 5, 20])
def test_pagerank_on_multigraph(iters):
    off, col, _ = multigraph()
    n, dmp = len(off) - 1, 0.85
    P = np.zeros((n, n))
    for u in range(n):
        deg = off[u + 1] - off[u]
        if deg == 0:
            P[u, :] = 1.0 / n
        for v in col[off[u]:off[u + 1]]:
            P[u, v] += 1.0 / deg          # multiplicity counts (R8)
    x = np.full(n, 1.0 / n)
    for _ in range(iters):
        x = x @ (dmp * P + (1 - dmp) / n)
    got = oracle.pagerank(off, col, dmp, iters)
    assert np.max(np.abs(got - x) / x) < 1e-13
    assert abs(got.sum() - 1.0) < 1e-12


def test_stage1_locality_counts_occurrences():
    off, col, _ = multigraph()
    n, S, B, M, A = len(off) - 1, 2, 2, 2, 0
    tp, mem = oracle.sample_tiles(off, col, B, M, A)
    loc1 = np.zeros(n, dtype=np.int64)
    for t in range(len(tp) - 1):
        T = mem[tp[t]:tp[t + 1]].tolist()
        for i, v in enumerate(T):
            loc1[v] += sum(1 for j, x in enumerate(T) if j != i and x // S == v // S)
    st = oracle.reorder_stages(n, tp, mem, S)
    assert np.array_equal(st["loc1"], loc1)
    # the sample itself: every tile<2> of every row (row 6 = [0,6 | 6,1 | 1,1])
    assert [mem[tp[t]:tp[t + 1]].tolist() for t in range(len(tp) - 1)] == \
        [[1, 1], [0, 2], [2, 2], [0, 3], [3, 3], [4, 4], [0, 6], [6, 1], [1, 1]]
