"""The multi-GPU path (1D partition) with p = 2, 3, 4 LOGICAL ranks on one GPU.

The test pool has one GPU per box, so the NCCL path can only run with world = 1, where no vertex
has a remote owner.  sage_debug_loopback_id (test-only, include/sage.h) swaps NCCL for a loopback
transport (xport.h): p graphs in one process, one host thread per rank, the collectives done as
stream-ordered device copies / reductions between the ranks' buffers.  Everything else — k_mpush
with remote owners, the padded indexing for r > 0, the sparse (C1a) and dense (C1b) exchanges,
k_mapply / k_mapply_sparse, the fused exchange over peer memory (exchange = 0: k_mpush ORs remote
candidates straight into the owner's inbox, on one GPU every rank's buffer is addressable), the pull
allgather, the SSSP min reduce-scatter and k_msssp_apply, the
PageRank reduce-scatter, the parent post-pass — is the product code.  The gathered slices must
equal the oracle's result (BFS / SSSP bit-exact, PageRank <= 1e-6 relative).
"""
import threading

import numpy as np
import pytest

import oracle
import sagegen as sg

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(900)]


@pytest.fixture(scope="module")
def sage():
    import torch
    assert torch.cuda.is_available()
    from __graft_entry__ import build
    build()
    import paper_conf_sigmod_00020t21_b200 as s
    return s


def blocks(n, p, skew=False):
    if not skew:
        return [(n * r // p, n * (r + 1) // p) for r in range(p)]
    cuts = [0] + sorted({max(1, min(n - 1, int(n * f))) for f in np.linspace(0.05, 0.9, p - 1)}) + [n]
    return list(zip(cuts[:-1], cuts[1:]))


def run_ranks(sage, g, w, p, fn, skew=False, **kw):
    """Load rank r's block on thread r (loopback transport), call fn(G, r) on every rank
    concurrently, return the per-rank results in rank order."""
    uid = sage.debug_loopback_id(p)
    bl = blocks(g.n, p, skew)
    out, errs = [None] * p, []

    def worker(r):
        vb, ve = bl[r]
        b0, b1 = int(g.off[vb]), int(g.off[ve])
        try:
            G = sage.load_csr(g.off[vb:ve + 1] - b0, g.col[b0:b1], None if w is None else w[b0:b1], n=g.n,
                              symmetric=g.symmetric, rank=r, world=p, nccl_unique_id=uid, v_begin=vb,
                              v_end=ve, **kw)
            try:
                out[r] = fn(G, r)
            finally:
                G.free()
        except Exception as e:      # noqa: BLE001 — re-raised below
            errs.append((r, e))

    ts = [threading.Thread(target=worker, args=(r,)) for r in range(p)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(600)
    assert not any(t.is_alive() for t in ts), "a rank hung"
    if errs:
        raise errs[0][1]
    return out


def _parents_ok(g, lv, par, s):
    assert par[s] == -1
    ok = lv > 0
    v = np.nonzero(ok)[0]
    p = par[ok]
    assert np.all(lv[p] == lv[v] - 1)
    for x, y in zip(p[:2000], v[:2000]):
        assert y in g.col[g.off[x]:g.off[x + 1]]


@pytest.mark.parametrize("exchange", [0, 1])
@pytest.mark.parametrize("p", [2, 3, 4])
@pytest.mark.parametrize("sym", [True, False])
def test_loopback_bfs(sage, p, sym, exchange):
    g = sg.rmat(14, 16, seed=3, symmetric=sym)
    srcs = [int(s) for s in sg.sources(g, 3, seed=2)]

    def fn(G, r):
        assert G.peer_exchange == (exchange == 0)
        res = []
        for s in srcs:
            for po in ((True, False) if sym else (True,)):
                lv, par, st = G.bfs(s, push_only=po, parents=True)
                res.append((s, po, lv.copy(), par.copy(), st))
        return res

    out = run_ranks(sage, g, None, p, fn, skew=(p == 3), exchange=exchange)
    for k in range(len(out[0])):
        s, po = out[0][k][0], out[0][k][1]
        lv = np.concatenate([o[k][2] for o in out])
        par = np.concatenate([o[k][3] for o in out])
        ref = oracle.bfs(g.off, g.col, s)
        assert np.array_equal(lv, ref), (p, sym, s, po)
        assert np.all(par[ref <= 0] == -1)
        _parents_ok(g, lv, par, s)
        st = out[0][k][4]
        assert st["edges_traversed"] == int(np.diff(g.off)[ref >= 0].sum()) // (2 if sym else 1)


@pytest.mark.parametrize("exchange", [0, 1])
def test_loopback_bfs_long_path_sparse_levels(sage, exchange):
    """A UK-like graph (crawl order, tendrils): hundreds of tiny levels, sparse exchange (or the
    peer inboxes), remote discoveries on block boundaries."""
    uk = sg.uk_like(n=60000, seed=1, n_tendrils=20, tmin=30, tmax=120, hmax=1 << 10)
    srcs = [int(s) for s in sg.sources(uk, 2, seed=2)]
    out = run_ranks(sage, uk, None, 4, lambda G, r: [G.bfs(s, push_only=True)[0].copy() for s in srcs],
                    exchange=exchange)
    for k, s in enumerate(srcs):
        lv = np.concatenate([o[k] for o in out])
        assert np.array_equal(lv, oracle.bfs(uk.off, uk.col, s))


@pytest.mark.parametrize("exchange", [0, 1])
@pytest.mark.parametrize("p", [2, 3])
@pytest.mark.parametrize("sym", [True, False])
def test_loopback_sssp(sage, p, sym, exchange):
    g = sg.rmat(13, 16, seed=5, symmetric=sym)
    w = sg.weights(g, 1)
    srcs = [int(s) for s in sg.sources(g, 3, seed=2)]
    out = run_ranks(sage, g, w, p, lambda G, r: [G.sssp(s)[0].copy() for s in srcs], exchange=exchange)
    for k, s in enumerate(srcs):
        d = np.concatenate([o[k] for o in out])
        assert np.array_equal(d, oracle.sssp(g.off, g.col, w, s)[0]), (p, sym, s)


def test_loopback_sssp_overflow(sage):
    n = 6
    off = np.array([0, 1, 2, 3, 4, 5, 5], dtype=np.int64)
    col = np.array([1, 2, 3, 4, 5], dtype=np.int32)
    w = np.array([0x70000000] * 5, dtype=np.uint32)
    g = sg.Graph(n=n, off=off, col=col, symmetric=False)

    def fn(G, r):
        try:
            G.sssp(0)
        except sage.SageError as e:
            return e.status
        return 0

    assert run_ranks(sage, g, w, 3, fn) == [sage.E_OVERFLOW] * 3
    assert run_ranks(sage, g, w, 3, fn, exchange=1) == [sage.E_OVERFLOW] * 3


def test_loopback_mixed_queries_peer_form(sage):
    """BFS and SSSP alternating on the same graphs in the peer form: each query resets only its
    own part of the shared peer region, so neither may leak into the other."""
    g = sg.rmat(12, 16, seed=9, symmetric=True)
    w = sg.weights(g, 3)
    srcs = [int(s) for s in sg.sources(g, 3, seed=4)]

    def fn(G, r):
        assert G.peer_exchange
        res = []
        for s in srcs:
            res.append(G.bfs(s, push_only=True)[0].copy())
            res.append(G.sssp(s)[0].copy())
        return res

    out = run_ranks(sage, g, w, 3, fn)
    for k, s in enumerate(srcs):
        assert np.array_equal(np.concatenate([o[2 * k] for o in out]), oracle.bfs(g.off, g.col, s))
        assert np.array_equal(np.concatenate([o[2 * k + 1] for o in out]), oracle.sssp(g.off, g.col, w, s)[0])


@pytest.mark.parametrize("p", [2, 3])
@pytest.mark.parametrize("sym", [True, False])
def test_loopback_pagerank(sage, p, sym):
    g = sg.rmat(13, 16, seed=7, symmetric=sym)
    out = run_ranks(sage, g, None, p, lambda G, r: G.pagerank(0.85, 20)[0].copy())
    x = np.concatenate(out)
    xr = oracle.pagerank(g.off, g.col, 0.85, 20)
    assert np.max(np.abs(x - xr) / xr) <= 1e-6
