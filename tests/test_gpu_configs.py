"""GPU parity on the shapes of BASELINE.json configs[2] and configs[3] at test sizes.

* twitter-like (C3 shape: directed, Zipf out-degree hubs, planted communities, scrambled ids):
  BFS, SSSP and PageRank equal the oracle; Sampling-based Reordering rounds give the oracle's
  permutation and relabelled CSR exactly, and answers in original ids are unchanged (C3 is the
  "reordering on vs off" config).
* UK-like (C4 shape: directed, crawl order, host blocks, tendril chains): more than 500 BFS levels
  in one persistent launch (device-resident level loop), PageRank, and the NCCL path's
  host-sequenced level loop.
"""
import numpy as np
import pytest

import oracle
import sagegen as sg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sage():
    import torch
    assert torch.cuda.is_available()
    from __graft_entry__ import build
    build()
    import paper_conf_sigmod_00020t21_b200 as s
    return s


@pytest.fixture(scope="module")
def tw():
    g = sg.twitter_like(n=60000, tuples=2_000_000, seed=1, cmin=8, cmax=4096)
    g.w = sg.weights(g, 4)
    return g


@pytest.fixture(scope="module")
def uk():
    return sg.uk_like(n=300000, seed=1, n_tendrils=40, tmin=100, tmax=600, hmax=1 << 14)


def test_twitter_like_queries(sage, tw):
    with sage.load_csr(tw.off, tw.col, tw.w) as G:
        for s in sg.sources(tw, 3, seed=2):
            s = int(s)
            lv, _, st = G.bfs(s)
            assert np.array_equal(lv, oracle.bfs(tw.off, tw.col, s))
            assert st["pull_levels"] == 0            # directed -> push only
            d, _ = G.sssp(s)
            assert np.array_equal(d, oracle.sssp(tw.off, tw.col, tw.w, s)[0])
        x, _ = G.pagerank(0.85, 20)
        xr = oracle.pagerank(tw.off, tw.col, 0.85, 20)
        assert np.max(np.abs(x - xr) / xr) <= 1e-6


def test_twitter_like_reorder_on_off(sage, tw):
    off2, col2, w2, sigma, info = oracle.reorder(tw.off, tw.col, tw.w, rounds=2)
    with sage.load_csr(tw.off, tw.col, tw.w) as G:
        before = G.objective(8)
        assert before == info[0]["objective_before"]
        srcs = [int(s) for s in sg.sources(tw, 2, seed=3)]
        pre = [G.bfs(s)[0] for s in srcs]
        st = G.reorder(2)
        assert st["levels"] == len(info) and st["vertices_discovered"] == sum(i["swaps"] for i in info)
        assert np.array_equal(G.permutation(), sigma)
        o, c, w = G.csr()
        assert np.array_equal(o, off2) and np.array_equal(c, col2) and np.array_equal(w, w2)
        assert G.objective(8) == oracle.objective(off2, col2)
        for s, p in zip(srcs, pre):
            lv, _, _ = G.bfs(s)
            assert np.array_equal(lv, p)
            d, _ = G.sssp(s)
            assert np.array_equal(d, oracle.sssp(tw.off, tw.col, tw.w, s)[0])


def test_uk_like_high_diameter(sage, uk):
    with sage.load_csr(uk.off, uk.col) as G:
        for s in sg.sources(uk, 2, seed=2):
            s = int(s)
            ref = oracle.bfs(uk.off, uk.col, s)
            lv, _, st = G.bfs(s)
            assert np.array_equal(lv, ref)
            assert st["levels"] == ref.max() + 1 and st["levels"] > 500
        x, _ = G.pagerank(0.85, 20)
        xr = oracle.pagerank(uk.off, uk.col, 0.85, 20)
        assert np.max(np.abs(x - xr) / xr) <= 1e-6


def test_uk_like_nccl_level_loop(sage, uk):
    s = int(sg.sources(uk, 1, seed=4)[0])
    with sage.load_csr(uk.off, uk.col, rank=0, world=1, nccl_unique_id=sage.nccl_unique_id()) as G:
        lv, _, st = G.bfs(s)
        assert np.array_equal(lv, oracle.bfs(uk.off, uk.col, s))
        assert st["levels"] > 500
