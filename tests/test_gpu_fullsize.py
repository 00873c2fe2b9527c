"""Parity at BASELINE.json's full single-GPU size (configs[1]: RMAT scale 24, symmetrised,
weights in [1, 255]) in the launch configuration bench.py times (persistent kernels, default
ladder B=256 M=8 A=4).

* BFS: levels equal the oracle's exactly (full serial BFS, a few seconds per source), push-only
  and direction-optimising.
* SSSP: the exact certificate of SURVEY §8(c) c2 (dist(s)=0, no arc can be relaxed, every reached
  vertex has a tight in-arc) — it accepts iff dist is the true shortest-distance vector.
* PageRank: the full 20-iteration oracle run (fp64, serial) vs the GPU's pull (default on this
  symmetric graph) and push (Alg. 1) forms, within 1e-6 relative at every vertex; and x_20 equals
  one oracle step applied to the GPU's x_19.
* Reorder: after one round, BFS answers in original ids are unchanged.
"""
import numpy as np
import pytest

import oracle
import sagegen as sg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def c2():
    return sg.config("C2")


@pytest.fixture(scope="module")
def G(c2):
    import torch
    from __graft_entry__ import build
    build()
    import paper_conf_sigmod_00020t21_b200 as sage
    g = sage.load_csr(torch.from_numpy(c2.off).cuda(), torch.from_numpy(c2.col).cuda(),
                      torch.from_numpy(c2.w).cuda(), symmetric=True, borrow=True)
    yield g
    g.free()


def test_c2_bfs_exact(c2, G):
    for s in sg.sources(c2, 2, seed=2):
        ref = oracle.bfs(c2.off, c2.col, int(s))
        lv, _, st = G.bfs(int(s), push_only=True)
        assert np.array_equal(lv, ref)
        assert st["arcs_inspected"] == int(np.diff(c2.off)[ref >= 0].sum())
        lv2, par, st2 = G.bfs(int(s), parents=True)
        assert np.array_equal(lv2, ref)
        assert st2["pull_levels"] >= 1
        ok = lv2 > 0
        assert np.all(ref[par[ok]] == ref[ok] - 1)


def test_c2_sssp_certificate(c2, G):
    s = int(sg.sources(c2, 1, seed=2)[0])
    d, st = G.sssp(s)
    assert oracle.check_sssp(c2.off, c2.col, c2.w, s, d) == 0
    assert st["levels"] > 5


def test_c2_pagerank_full_oracle(c2, G):
    ref = oracle.pagerank(c2.off, c2.col, 0.85, 20)
    for po in (False, True):
        x, _ = G.pagerank(0.85, 20, push_only=po)
        assert np.max(np.abs(x - ref) / ref) <= 1e-6, po


def test_c2_pagerank_step_property(c2, G):
    x19, _ = G.pagerank(0.85, 19)
    x20, _ = G.pagerank(0.85, 20)
    ref = oracle.pagerank_step(c2.off, c2.col, x19, 0.85)
    assert np.max(np.abs(x20 - ref) / ref) <= 1e-6
    assert abs(x20.sum() - 1.0) < 1e-9


def test_c2_reorder_keeps_bfs(c2):
    import torch
    import paper_conf_sigmod_00020t21_b200 as sage
    s = int(sg.sources(c2, 1, seed=5)[0])
    ref = oracle.bfs(c2.off, c2.col, s)
    with sage.load_csr(torch.from_numpy(c2.off).cuda(), torch.from_numpy(c2.col).cuda(), symmetric=True) as H:
        before = H.objective(8)
        st = H.reorder(1)
        assert st["vertices_discovered"] > 0 and H.objective(8) < before
        lv, _, _ = H.bfs(s, push_only=True)
        assert np.array_equal(lv, ref)
        perm = H.permutation()
        assert np.array_equal(np.sort(perm), np.arange(c2.n, dtype=np.int32))


def test_c2_bc_one_source(c2, G):
    """NEXT #1 at full size: one source's Brandes dependencies vs the serial oracle."""
    s = sg.sources(c2, 1, seed=6)
    got, st = G.bc(s)
    ref = oracle.bc(c2.off, c2.col, s)
    tol = 1e-9 * np.max(np.abs(ref)) + 1e-6 * np.abs(ref)
    assert np.all(np.abs(got - ref) <= tol)
