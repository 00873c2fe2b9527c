"""Out-of-core traversal: columns and weights in pinned,
mapped host memory, read zero-copy by the same kernels.  Results must equal the oracle."""
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


@pytest.mark.parametrize("borrow", [False, True])
@pytest.mark.parametrize("align", [4, 32, 0])
def test_host_columns_parity(sage, borrow, align):
    g = sg.rmat(14, 16, seed=51, symmetric=True)
    w = sg.weights(g, 2)
    col, ww = g.col.copy(), w.copy()
    with sage.load_csr(g.off, col, ww, symmetric=True, host_columns=True, borrow=borrow, align=align) as G:
        for s in sg.sources(g, 2, seed=2):
            s = int(s)
            ref = oracle.bfs(g.off, g.col, s)
            for po in (True, False):
                assert np.array_equal(G.bfs(s, push_only=po)[0], ref)
            assert np.array_equal(G.sssp(s)[0], oracle.sssp(g.off, g.col, w, s)[0])
        x, _ = G.pagerank(0.85, 10)
        assert np.max(np.abs(x - oracle.pagerank(g.off, g.col, 0.85, 10)) / x) <= 1e-6
        with pytest.raises(sage.SageError) as ei:
            G.reorder(1)
        assert ei.value.status == sage.E_UNSUPPORTED


def test_host_columns_directed_uk_shape(sage):
    g = sg.uk_like(n=200000, seed=3, n_tendrils=20, tmin=50, tmax=200, hmax=1 << 12)
    with sage.load_csr(g.off, g.col, host_columns=True, align=32) as G:
        s = int(sg.sources(g, 1, seed=2)[0])
        assert np.array_equal(G.bfs(s)[0], oracle.bfs(g.off, g.col, s))
