"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every
product kernel family on RMAT-12 (BFS push + DO with the fused tiling and the hub filter forced
on, SSSP, PageRank pull / push / windowed push, a reorder round, BC), results checked against the
oracle so a sanitizer run that perturbs timing still has to produce the right answers."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

g = sg.rmat(12, 16, seed=1, symmetric=True)
w = sg.weights(g, 1)
s = int(sg.sources(g, 1, seed=2)[0])
ref = oracle.bfs(g.off, g.col, s)
with sage.load_csr(g.off, g.col, w, symmetric=True, hub_filter=1) as G:
    for po in (True, False):
        lv, par, _ = G.bfs(s, push_only=po, parents=True)
        assert np.array_equal(lv, ref)
    d, _ = G.sssp(s)
    assert np.array_equal(d, oracle.sssp(g.off, g.col, w, s)[0])
    xr = oracle.pagerank(g.off, g.col, 0.85, 5)
    for po in (False, True):
        x, _ = G.pagerank(0.85, 5, push_only=po)
        assert np.max(np.abs(x - xr) / xr) <= 1e-6
    G.reorder(1)
    assert np.array_equal(G.bfs(s, push_only=True)[0], ref)
    b, _ = G.bc([s])
    br = oracle.bc(g.off, g.col, [s])
    assert np.all(np.abs(b - br) <= 1e-9 * np.max(np.abs(br)) + 1e-6 * np.abs(br))
# windowed push PageRank (chosen on a crawl-ordered UK-like graph)
uk = sg.uk_like(n=200000, seed=1, n_tendrils=10, tmin=20, tmax=40, hmax=1 << 12)
with sage.load_csr(uk.off, uk.col) as G:
    x, _ = G.pagerank(0.85, 3)
    assert G.pagerank_windowed
    xr = oracle.pagerank(uk.off, uk.col, 0.85, 3)
    assert np.max(np.abs(x - xr) / xr) <= 1e-6
print("sanitize workload ok")
