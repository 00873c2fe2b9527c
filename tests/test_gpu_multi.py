"""The NCCL multi-GPU path (1D partition) on a 1-rank communicator.

gpurun and the round-end runs expose one GPU, so world > 1 cannot run on NCCL here; with
dist != NULL and world == 1 the library takes exactly the host-sequenced NCCL path (padded layout,
per-level stats allreduce, frontier allgather before pull levels, PR reduce-scatter).  World 2-4
runs on one GPU through the loopback transport in tests/test_gpu_multi_loopback.py, and the
protocol is modelled on CPU with gloo in tests/test_partition_model.py.
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


@pytest.mark.parametrize("sym", [True, False])
def test_nccl_path_bfs_pagerank(sage, sym):
    g = sg.rmat(14, 16, seed=3, symmetric=sym)
    uid = sage.nccl_unique_id()
    with sage.load_csr(g.off, g.col, symmetric=sym, rank=0, world=1, nccl_unique_id=uid,
                       v_begin=0, v_end=g.n) as G:
        for s in sg.sources(g, 4, seed=2):
            ref = oracle.bfs(g.off, g.col, int(s))
            for po in (True, False):
                lv, _, st = G.bfs(int(s), push_only=po)
                assert np.array_equal(lv, ref)
                assert st["edges_traversed"] == int(np.diff(g.off)[ref >= 0].sum()) // (2 if sym else 1)
            if sym:
                assert st["pull_levels"] >= 1
        x, _ = G.pagerank(0.85, 20)
        xr = oracle.pagerank(g.off, g.col, 0.85, 20)
        assert np.max(np.abs(x - xr) / xr) <= 1e-6
        s = int(sg.sources(g, 1, seed=4)[0])
        lv, par, _ = G.bfs(s, parents=True)       # parents on the multi-GPU path (post-pass)
        ref = oracle.bfs(g.off, g.col, s)
        assert par[s] == -1 and np.all(par[ref < 0] == -1)
        ok = ref > 0
        assert np.all(ref[par[ok]] == ref[ok] - 1)


@pytest.mark.parametrize("sym", [True, False])
def test_nccl_path_sssp(sage, sym):
    """Multi-GPU SSSP (NEXT #2) through the 1-rank NCCL path: bit-exact vs Dijkstra."""
    g = sg.rmat(13, 16, seed=5, symmetric=sym)
    w = sg.weights(g, 1)
    uid = sage.nccl_unique_id()
    with sage.load_csr(g.off, g.col, w, symmetric=sym, rank=0, world=1, nccl_unique_id=uid) as G:
        for s in sg.sources(g, 3, seed=2):
            d, st = G.sssp(int(s))
            ref, _ = oracle.sssp(g.off, g.col, w, int(s))
            assert np.array_equal(d, ref)
            assert st["edges_traversed"] == int(np.diff(g.off)[ref != 0xFFFFFFFF].sum()) // (2 if sym else 1)


def test_nccl_path_sssp_overflow(sage):
    """A path whose length exceeds UINT32_MAX is reported, as on one GPU."""
    off = np.array([0, 1, 2, 2], dtype=np.int64)
    col = np.array([1, 2], dtype=np.int32)
    w = np.array([0xF0000000, 0xF0000000], dtype=np.uint32)
    with sage.load_csr(off, col, w, rank=0, world=1, nccl_unique_id=sage.nccl_unique_id()) as G:
        with pytest.raises(sage.SageError) as ei:
            G.sssp(0)
        assert ei.value.status == sage.E_OVERFLOW
    # overflowing candidate that is not needed: 0->2 directly is short
    off = np.array([0, 2, 3, 3], dtype=np.int64)
    col = np.array([1, 2, 2], dtype=np.int32)
    w = np.array([0xF0000000, 5, 0xF0000000], dtype=np.uint32)
    with sage.load_csr(off, col, w, rank=0, world=1, nccl_unique_id=sage.nccl_unique_id()) as G:
        d, _ = G.sssp(0)
        assert d.tolist() == [0, 0xF0000000, 5]


def test_nccl_path_refuses_bad_blocks(sage):
    g = sg.rmat(10, 8, seed=1, symmetric=True)
    with pytest.raises(sage.SageError):
        sage.load_csr(g.off[:11], g.col[:g.off[10]], rank=0, world=1, nccl_unique_id=sage.nccl_unique_id(),
                      v_begin=0, v_end=10, n=g.n)   # one rank must cover [0, n)
