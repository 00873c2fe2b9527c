"""GPU parity of Betweenness Centrality (NEXT #1; Alg. 1 l.8-24) against the Brandes oracle.
Tolerance: |bc_gpu - bc_ora| <= 1e-9 * max(|bc_ora|) + 1e-6 * |bc_ora| (fp64 atomics reorder the
sums; sigma can reach ~1e30 on RMAT, so a purely absolute bound would be meaningless)."""
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


def _close(got, ref):
    tol = 1e-9 * max(np.max(np.abs(ref)), 1e-300) + 1e-6 * np.abs(ref)
    return np.all(np.abs(got - ref) <= tol)


@pytest.mark.parametrize("lad", [dict(), dict(tile_cta=16, tile_min=8, align=0)], ids=["default", "fig3"])
def test_bc_parity(sage, lad):
    graphs = [sg.random_graph(40, 150, seed=k, symmetric=bool(k % 2)) for k in range(4)]
    graphs += [sg.rmat(12, 16, seed=41, symmetric=True), sg.rmat(12, 16, seed=42, symmetric=False),
               sg.from_edges(8, [(0, i) for i in range(1, 8)], True, "star"),
               sg.from_edges(12, [(i, i + 1) for i in range(11)], False, "path")]
    for g in graphs:
        srcs = sg.sources(g, 4, seed=3)
        with sage.load_csr(g.off, g.col, symmetric=g.symmetric, **lad) as G:
            got, st = G.bc(srcs)
        ref = oracle.bc(g.off, g.col, srcs)
        assert _close(got, ref), (g.name, np.max(np.abs(got - ref)))


def test_bc_all_sources_small(sage):
    g = sg.rmat(9, 8, seed=7, symmetric=True)
    srcs = np.arange(g.n, dtype=np.int32)
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        got, _ = G.bc(srcs)
    assert _close(got, oracle.bc(g.off, g.col, srcs))


def test_bc_after_reorder(sage):
    g = sg.rmat(12, 16, seed=9, symmetric=True)
    srcs = sg.sources(g, 3, seed=2)
    ref = oracle.bc(g.off, g.col, srcs)
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        G.reorder(2)
        got, _ = G.bc(srcs)
    assert _close(got, ref)


def test_bc_rmat18(sage):
    g = sg.rmat(18, 16, seed=1, symmetric=True)
    srcs = sg.sources(g, 2, seed=2)
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        got, st = G.bc(srcs)
    assert _close(got, oracle.bc(g.off, g.col, srcs))
    assert st["levels"] >= 2
