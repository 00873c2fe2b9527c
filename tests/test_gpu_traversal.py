"""GPU parity of the CUDA path against the oracle (run on a B200 with -m gpu).

Bars (BASELINE.json north_star): BFS levels and SSSP distances bit-exact; PageRank within 1e-6
relative L-inf; the tile log (Tiled Partitioning, Alg. 2/3) equal to the oracle's as an exact
multiset.  BFS parents are not unique: they are checked by rule (level(p) = level(v) - 1 and the
arc p->v exists).  Every graph is seeded and synthetic.
"""
import numpy as np
import pytest

import oracle
import sagegen as sg

pytestmark = pytest.mark.gpu

LADDERS = [dict(tile_cta=256, tile_min=8, align=4),     # build default (int4 loads)
           dict(tile_cta=256, tile_min=8, align=0),     # paper mode: no alignment (scalar loads)
           dict(tile_cta=16, tile_min=8, align=0),      # Figure 3's ladder
           dict(tile_cta=1024, tile_min=4, align=32),
           dict(tile_cta=64, tile_min=1, align=0)]


@pytest.fixture(scope="module")
def sage():
    import torch
    assert torch.cuda.is_available()
    from __graft_entry__ import build
    build()
    import paper_conf_sigmod_00020t21_b200 as s
    return s


def _hand_graphs():
    gs = []
    gs.append(sg.from_edges(6, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5)], True, "path"))
    gs.append(sg.from_edges(9, [(0, i) for i in range(1, 9)], True, "star"))
    gs.append(sg.from_edges(7, [(i, (i + 1) % 7) for i in range(7)], False, "dcycle"))
    gs.append(sg.from_edges(6, [(i, j) for i in range(6) for j in range(6) if i != j], False, "complete"))
    gs.append(sg.from_edges(8, [(0, 1), (2, 3), (3, 4)], True, "disconnected"))
    gs.append(sg.from_edges(1, [], False, "single"))
    gs.append(sg.from_edges(40, [(0, i) for i in range(1, 40)] + [(i, i + 1) for i in range(1, 39)], False,
                            "fan+chain"))
    return gs


def _parents_ok(off, col, level, parent, src):
    n = len(level)
    assert parent[src] == -1
    for v in range(n):
        if level[v] <= 0:
            if v != src:
                assert parent[v] == -1 or level[v] == 0
            continue
        p = parent[v]
        assert 0 <= p < n and level[p] == level[v] - 1
        assert v in col[off[p]:off[p + 1]]


@pytest.mark.parametrize("push_only", [True, False])
def test_bfs_hand_graphs(sage, push_only):
    for g in _hand_graphs():
        with sage.load_csr(g.off, g.col, symmetric=g.symmetric) as G:
            for s in range(g.n):
                lv, par, _ = G.bfs(s, parents=True, push_only=push_only)
                assert np.array_equal(lv, oracle.bfs(g.off, g.col, s)), (g.name, s)
                _parents_ok(g.off, g.col, lv, par, s)


@pytest.mark.parametrize("lad", LADDERS, ids=lambda d: f"B{d['tile_cta']}M{d['tile_min']}A{d['align']}")
def test_bfs_random_and_rmat(sage, lad):
    graphs = [sg.random_graph(50, 300, seed=k, symmetric=bool(k % 2)) for k in range(6)]
    graphs.append(sg.rmat(12, 16, seed=3, symmetric=True))
    graphs.append(sg.rmat(12, 16, seed=4, symmetric=False))
    for g in graphs:
        with sage.load_csr(g.off, g.col, symmetric=g.symmetric, **lad) as G:
            for s in sg.sources(g, 4, seed=2):
                for po in (True, False):
                    lv, _, st = G.bfs(int(s), push_only=po)
                    ref = oracle.bfs(g.off, g.col, int(s))
                    assert np.array_equal(lv, ref), (g.name, int(s), po)


def test_bfs_config1_all_sources(sage):
    """C1 (RMAT-16 symmetric, BASELINE configs[0]): 64 seeded sources, push-only and direction-optimising."""
    g = sg.config("C1")
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        for s in sg.sources(g, 64, seed=2):
            ref = oracle.bfs(g.off, g.col, int(s))
            for po in (True, False):
                lv, par, st = G.bfs(int(s), parents=True, push_only=po)
                assert np.array_equal(lv, ref)
                p = par[lv > 0]
                assert np.all(lv[p] == lv[lv > 0] - 1)
            reached = ref >= 0
            assert st["edges_traversed"] == int(np.diff(g.off)[reached].sum()) // 2
            if not po:
                pass


def test_bfs_direction_switch_actually_pulls(sage):
    g = sg.rmat(16, 16, seed=1, symmetric=True)
    s = int(sg.sources(g, 1, seed=2)[0])
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        _, _, st = G.bfs(s)
        assert st["pull_levels"] >= 1 and st["push_levels"] >= 1
        assert st["arcs_inspected"] < 0.5 * g.m
        _, _, st2 = G.bfs(s, push_only=True)
        assert st2["pull_levels"] == 0
        assert st2["arcs_inspected"] == int(np.diff(g.off)[oracle.bfs(g.off, g.col, s) >= 0].sum())


def test_bfs_device_buffers_and_borrow(sage):
    import torch
    g = sg.rmat(12, 8, seed=5, symmetric=True)
    off = torch.from_numpy(g.off).cuda()
    col = torch.from_numpy(g.col).cuda()
    with sage.load_csr(off, col, symmetric=True, borrow=True) as G:
        out = torch.empty(g.n, dtype=torch.int32, device="cuda")
        s = int(sg.sources(g, 1, seed=2)[0])
        G.bfs(s, out=out)
        assert np.array_equal(out.cpu().numpy(), oracle.bfs(g.off, g.col, s))


def test_unsorted_rows_and_unaligned_borrow(sage):
    import torch
    g = sg.rmat(11, 8, seed=6, symmetric=False)
    rng = np.random.default_rng(0)
    col = g.col.copy()
    for u in range(g.n):
        rng.shuffle(col[g.off[u]:g.off[u + 1]])
    # borrowed column array starting 4 bytes past a 16-B boundary -> scalar (VEC=1) path
    big = torch.zeros(len(col) + 1, dtype=torch.int32, device="cuda")
    big[1:] = torch.from_numpy(col).cuda()
    colv = big[1:]
    off = torch.from_numpy(g.off).cuda()
    with sage.load_csr(off, colv, borrow=True) as G:
        assert not G.rows_sorted
        for s in sg.sources(g, 3, seed=2):
            lv, _, _ = G.bfs(int(s))
            assert np.array_equal(lv, oracle.bfs(g.off, g.col, int(s)))


@pytest.mark.parametrize("lad", LADDERS[:3], ids=lambda d: f"B{d['tile_cta']}M{d['tile_min']}A{d['align']}")
def test_sssp_parity(sage, lad):
    graphs = [sg.random_graph(40, 200, seed=k, symmetric=bool(k % 2)) for k in range(4)]
    graphs.append(sg.rmat(12, 16, seed=7, symmetric=True))
    graphs.append(sg.rmat(12, 16, seed=8, symmetric=False))
    for g in graphs:
        w = sg.weights(g, 3)
        with sage.load_csr(g.off, g.col, w, symmetric=g.symmetric, **lad) as G:
            for s in sg.sources(g, 3, seed=2):
                d, st = G.sssp(int(s))
                ref, ovf = oracle.sssp(g.off, g.col, w, int(s))
                assert not ovf
                assert np.array_equal(d, ref), (g.name, int(s))


def test_sssp_unit_weights_equal_bfs(sage):
    g = sg.rmat(13, 16, seed=9, symmetric=True)
    w = np.ones(g.m, dtype=np.uint32)
    with sage.load_csr(g.off, g.col, w, symmetric=True) as G:
        s = int(sg.sources(g, 1, seed=2)[0])
        d, _ = G.sssp(s)
        lv, _, _ = G.bfs(s)
        lv64 = lv.astype(np.int64)
        assert np.array_equal(d.astype(np.int64), np.where(lv64 < 0, 2**32 - 1, lv64))


def test_sssp_overflow_and_near_overflow(sage):
    # path 0 -> 1 -> 2 with weights summing to exactly UINT32_MAX - 1 (valid) and one more hop (overflow)
    g = sg.from_edges(4, [(0, 1), (1, 2), (2, 3)], False, "p4")
    big = 2**31 - 1
    w = np.array([big, big, 5], dtype=np.uint32)      # d(2) = 2^32 - 2, d(3) overflows
    with sage.load_csr(g.off, g.col, w) as G:
        with pytest.raises(sage.SageError) as ei:
            G.sssp(0)
        assert ei.value.status == sage.E_OVERFLOW
    w2 = np.array([big, big, 1], dtype=np.uint32)     # d(3) = 2^32 - 1 = UINT32_MAX: also overflow (R4)
    with sage.load_csr(g.off, g.col, w2) as G:
        with pytest.raises(sage.SageError):
            G.sssp(0)
    g2 = sg.from_edges(3, [(0, 1), (1, 2)], False, "p3")
    with sage.load_csr(g2.off, g2.col, np.array([big, big], dtype=np.uint32)) as G:
        d, _ = G.sssp(0)
        ref, ovf = oracle.sssp(g2.off, g2.col, np.array([big, big], dtype=np.uint32), 0)
        assert not ovf and np.array_equal(d, ref) and d[2] == 2**32 - 2


@pytest.mark.parametrize("lad", LADDERS[:3], ids=lambda d: f"B{d['tile_cta']}M{d['tile_min']}A{d['align']}")
def test_pagerank_parity(sage, lad):
    graphs = [sg.random_graph(60, 300, seed=k, symmetric=bool(k % 2)) for k in range(3)]
    graphs.append(sg.rmat(13, 16, seed=1, symmetric=True))
    graphs.append(sg.rmat(13, 16, seed=2, symmetric=False))      # has dangling vertices
    graphs.append(sg.from_edges(5, [], False, "edgeless"))
    for g in graphs:
        with sage.load_csr(g.off, g.col, symmetric=g.symmetric, **lad) as G:
            for push_only in (True, False):      # push (Alg. 1) and, on symmetric graphs, pull
                for iters in (0, 1, 20):
                    x, st = G.pagerank(0.85, iters, push_only=push_only)
                    ref = oracle.pagerank(g.off, g.col, 0.85, iters)
                    assert np.max(np.abs(x - ref) / ref) <= 1e-6, (g.name, iters, push_only)
                    assert abs(x.sum() - 1.0) < 1e-6
            x2, _ = G.pagerank(0.85, 20)     # the resident log is reused across calls
            assert np.max(np.abs(x2 - oracle.pagerank(g.off, g.col, 0.85, 20)) / x2) <= 1e-6


@pytest.mark.parametrize("d", [0.5, 0.9, 0.95, 0.99])
def test_pagerank_damping_range(sage, d):
    """Pull (fp32 contributions up to d = 0.9, fp64 above) and push forms within 1e-6 of the
    oracle across the damping range the ABI accepts."""
    g = sg.rmat(16, 16, seed=13, symmetric=True)
    ref = oracle.pagerank(g.off, g.col, d, 30)
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        for po in (False, True):
            x, _ = G.pagerank(d, 30, push_only=po)
            assert np.max(np.abs(x - ref) / ref) <= 1e-6, (d, po)


def test_pagerank_pull_precision_at_scale(sage):
    """Pull form: fp32 contributions, fp64 accumulation (R7) stays well inside 1e-6 on RMAT-18."""
    g = sg.rmat(18, 16, seed=3, symmetric=True)
    with sage.load_csr(g.off, g.col, symmetric=True) as G:
        x, _ = G.pagerank(0.85, 20)
        xp, _ = G.pagerank(0.85, 20, push_only=True)
    ref = oracle.pagerank(g.off, g.col, 0.85, 20)
    assert np.max(np.abs(x - ref) / ref) <= 1e-6
    assert np.max(np.abs(xp - ref) / ref) <= 1e-12


@pytest.mark.parametrize("lad", LADDERS, ids=lambda d: f"B{d['tile_cta']}M{d['tile_min']}A{d['align']}")
def test_tile_log_equals_oracle(sage, lad):
    """c4: the device classifier's resident tile log == the oracle's decomposition (exact multiset)."""
    g = sg.rmat(14, 16, seed=11, symmetric=False)
    verts = np.arange(g.n, dtype=np.int32)
    with sage.load_csr(g.off, g.col, **lad) as G:
        got = G.export_tiles(verts)
    ref = oracle.tile_log(g.off, verts, lad["tile_cta"], lad["tile_min"], lad["align"])
    key = lambda a: a[np.lexsort((a[:, 3], a[:, 2], a[:, 1], a[:, 0]))]
    assert got.shape == ref.shape
    assert np.array_equal(key(got), key(ref))


def test_figure3_on_device(sage, golden_dir):
    import json
    import os
    fx = json.load(open(os.path.join(golden_dir, "fig3_tiles.json")))
    # one vertex per Figure 3 row, each row starting at offset 0 of its own graph
    for row in fx["rows"]:
        d = row["end"] - row["begin"]
        g = sg.from_edges(d + 1, [(0, j) for j in range(1, d + 1)], False, row["color"])
        with sage.load_csr(g.off, g.col, tile_cta=fx["B"], tile_min=fx["M"], align=fx["A"]) as G:
            got = sorted(tuple(int(x) for x in q[1:]) for q in G.export_tiles([0]))
        assert got == sorted(tuple(t) for t in row["tiles"]), row["color"]


def test_error_conventions(sage):
    g = sg.rmat(8, 4, seed=1)
    with sage.load_csr(g.off, g.col) as G:
        with pytest.raises(sage.SageError) as ei:
            G.bfs(g.n)
        assert ei.value.status == sage.E_INVALID
        with pytest.raises(sage.SageError) as ei:
            G.sssp(0)                                   # no weights
        assert ei.value.status == sage.E_INVALID
        with pytest.raises(sage.SageError) as ei:
            G.pagerank(1.0, 20)
        assert ei.value.status == sage.E_INVALID
        lv, _, _ = G.bfs(int(sg.sources(g, 1)[0]))      # graph still usable
    bad = g.col.copy()
    bad[3] = g.n
    with pytest.raises(sage.SageError) as ei:
        sage.load_csr(g.off, bad)
    assert ei.value.status == sage.E_INVALID
    w0 = np.ones(g.m, dtype=np.uint32)
    w0[5] = 0
    with pytest.raises(sage.SageError):
        sage.load_csr(g.off, g.col, w0)
    off2 = g.off.copy()
    off2[10] = off2[11] + 1
    with pytest.raises(sage.SageError):
        sage.load_csr(off2, g.col)
    with pytest.raises(sage.SageError):
        sage.load_csr(g.off, g.col, tile_cta=100)


def test_push_parity_multi_slice_and_skewed(sage):
    """Push and direction-optimising BFS on graphs above 2^20 vertices, and on a skewed graph whose
    arcs all target the first 2^20 vertices: the oracle's levels."""
    graphs = [sg.rmat(12, 16, seed=21, symmetric=True), sg.rmat(21, 8, seed=22, symmetric=True),
              sg.rmat(21, 8, seed=23, symmetric=False)]
    for g in graphs:
        with sage.load_csr(g.off, g.col, symmetric=g.symmetric) as G:
            for s in sg.sources(g, 2, seed=2):
                ref = oracle.bfs(g.off, g.col, int(s))
                for po in (True, False):
                    lv, _, st = G.bfs(int(s), push_only=po)
                    assert np.array_equal(lv, ref), (g.name, int(s), po)
    n = 3 << 20
    rng = np.random.default_rng(5)
    src = rng.integers(0, n, size=400000)
    dst = rng.integers(0, 1 << 20, size=400000)
    chain = np.stack([np.arange(0, 1 << 20), np.arange(1, (1 << 20) + 1)], 1)   # connect slice 0
    e = np.concatenate([np.stack([src, dst], 1), np.stack([dst, src], 1), chain])
    g = sg.from_edges(n, e, False, "skewed")
    with sage.load_csr(g.off, g.col) as G:
        for s in [int(src[0]), 0]:
            ref = oracle.bfs(g.off, g.col, s)
            lv, _, _ = G.bfs(s, push_only=True)
            assert np.array_equal(lv, ref)


def test_no_stealing_ablation_parity(sage):
    """SAGE_F_NO_STEALING (static tile assignment, the Fig. 10 ablation) gives the same levels."""
    for g in [sg.rmat(14, 16, seed=31, symmetric=True), sg.rmat(13, 16, seed=32, symmetric=False)]:
        with sage.load_csr(g.off, g.col, symmetric=g.symmetric) as G:
            for s in sg.sources(g, 3, seed=2):
                ref = oracle.bfs(g.off, g.col, int(s))
                lv, _, _ = G.bfs(int(s), push_only=True, stealing=False)
                assert np.array_equal(lv, ref)
    g = sg.rmat(13, 16, seed=33, symmetric=True)
    with sage.load_csr(g.off, g.col, symmetric=True, tile_cta=4096, tile_min=4096, align=0) as G:
        s = int(sg.sources(g, 1, seed=2)[0])
        assert np.array_equal(G.bfs(s, push_only=True)[0], oracle.bfs(g.off, g.col, s))


def test_pagerank_push_parity_repeat_and_reorder(sage):
    """Push PageRank (Alg. 1 l.26-29) within 1e-6 of the oracle on directed and symmetric inputs,
    repeated calls (the resident log is reused) and after a reorder (log rebuilt for the new
    labels), and on a UK-like (crawl order, tendrils) graph."""
    for sym, seed in ((False, 3), (True, 4)):
        g = sg.rmat(15, 16, seed=seed, symmetric=sym)
        xr = oracle.pagerank(g.off, g.col, 0.85, 20)
        with sage.load_csr(g.off, g.col, symmetric=sym) as G:
            for _ in range(2):
                x, _ = G.pagerank(0.85, 20, push_only=True)
                assert np.max(np.abs(x - xr) / xr) <= 1e-6
            G.reorder(rounds=1)
            x, _ = G.pagerank(0.85, 20, push_only=True)
            assert np.max(np.abs(x - xr) / xr) <= 1e-6
    uk = sg.uk_like(n=200000, seed=1, n_tendrils=10, tmin=20, tmax=60, hmax=1 << 12)
    xr = oracle.pagerank(uk.off, uk.col, 0.85, 10)
    with sage.load_csr(uk.off, uk.col) as G:
        x, _ = G.pagerank(0.85, 10)
        assert np.max(np.abs(x - xr) / xr) <= 1e-6


def test_full_occupancy_grid_on_small_graphs(sage):
    """Small graphs run the persistent kernels with one CTA per SM by default; the full-occupancy
    grid (sage_options.ctas_per_sm = 4, the configuration of the large configs) gives the same
    answers."""
    g = sg.rmat(15, 16, seed=9, symmetric=True)
    w = sg.weights(g, 1)
    with sage.load_csr(g.off, g.col, w, symmetric=True, ctas_per_sm=4) as G:
        for s in sg.sources(g, 4, seed=2):
            ref = oracle.bfs(g.off, g.col, int(s))
            for po in (True, False):
                assert np.array_equal(G.bfs(int(s), push_only=po)[0], ref)
            d, _ = G.sssp(int(s))
            assert np.array_equal(d, oracle.sssp(g.off, g.col, w, int(s))[0])
        x, _ = G.pagerank(0.85, 10)
        xr = oracle.pagerank(g.off, g.col, 0.85, 10)
        assert np.max(np.abs(x - xr) / xr) <= 1e-6


def test_deferred_contraction_every_level(sage):
    """Push BFS / SSSP with the deferred frontier list + K2' phase on every level: exact."""
    for sym in (True, False):
        g = sg.rmat(14, 16, seed=12, symmetric=sym)
        w = sg.weights(g, 1)
        with sage.load_csr(g.off, g.col, w, symmetric=sym) as G:
            for s in sg.sources(g, 3, seed=2):
                assert np.array_equal(G.bfs(int(s), push_only=True)[0], oracle.bfs(g.off, g.col, int(s)))
                assert np.array_equal(G.sssp(int(s))[0], oracle.sssp(g.off, g.col, w, int(s))[0])


@pytest.mark.parametrize("scale,sym", [(14, True), (16, True), (16, False), (18, True)])
def test_hub_filter_parity(sage, scale, sym):
    """Push BFS with the shared-memory hub filter forced on (8-bit keys, n <= 2^24) equals the
    oracle's levels and, with parents, passes the parent rule; with the filter forced off too."""
    g = sg.rmat(scale, 16, seed=40 + scale, symmetric=sym)
    for hub in (1, -1):
        with sage.load_csr(g.off, g.col, symmetric=sym, hub_filter=hub) as G:
            for s in sg.sources(g, 3, seed=2):
                ref = oracle.bfs(g.off, g.col, int(s))
                lv, par, _ = G.bfs(int(s), push_only=True, parents=True)
                assert np.array_equal(lv, ref), (hub, int(s))
                _parents_ok(g.off, g.col, lv, par, int(s))
                lv, _, _ = G.bfs(int(s))
                assert np.array_equal(lv, ref), (hub, int(s), "do")


def test_hub_filter_16bit_keys(sage):
    """n > 2^24 selects 16-bit hub keys: a sparse random graph over 2^24 + 5000 vertices with a
    dense core (hubs) gives the oracle's levels."""
    n = (1 << 24) + 5000
    rng = np.random.default_rng(7)
    core = rng.integers(0, n, size=2000)
    src = rng.integers(0, n, size=3_000_000)
    dst = core[rng.integers(0, len(core), size=3_000_000)]
    e = np.stack([src, dst], 1)
    g = sg.from_edges(n, np.concatenate([e, e[:, ::-1]]), True, "hubby")
    with sage.load_csr(g.off, g.col, symmetric=True, hub_filter=1) as G:
        for s in [int(core[0]), int(src[1])]:
            ref = oracle.bfs(g.off, g.col, s)
            lv, _, _ = G.bfs(s, push_only=True)
            assert np.array_equal(lv, ref)


def _banded_graph(n=120000, seed=7):
    """Directed graph whose arcs mostly stay near their source: offsets at and around the windowed
    push's halo (4096) and chunk (8192) boundaries, empty rows, long rows (> 32 and > 128 arcs in
    one 32-row group) and a few far arcs.  Duplicate arcs and self-loops are kept (R8)."""
    rng = np.random.default_rng(seed)
    offs = np.array([0, 1, -1, 2, 31, -32, 4095, -4095, 4096, -4096, 4097, 8191, 8192, -8193, 12287])
    rows = []
    for u in range(n):
        k = int(rng.integers(0, 6))
        if u % 997 == 0:
            k = 300
        if u % 13 == 0:
            k = 0
        t = u + rng.choice(offs, size=k)
        far = rng.random(k) < 0.1
        t[far] = rng.integers(0, n, size=int(far.sum()))
        rows.append(np.clip(t, 0, n - 1))
    deg = np.array([len(r) for r in rows], dtype=np.int64)
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(deg)
    col = np.concatenate(rows).astype(np.int32)
    return off, col


@pytest.mark.gpu
def test_pagerank_windowed_push(sage):
    """Windowed push PageRank (shared-memory accumulation of near targets) vs the
    oracle on graphs that select it: a banded multigraph with targets on the halo / chunk
    boundaries, and a UK-like crawl-order graph; the log-based push (stealing off) agrees."""
    off, col = _banded_graph()
    uk = sg.uk_like(n=300000, seed=2, n_tendrils=20, tmin=20, tmax=80, hmax=1 << 14)
    for o, c in ((off, col), (uk.off, uk.col)):
        for d, it in ((0.85, 20), (0.99, 7)):
            xr = oracle.pagerank(o, c, d, it)
            with sage.load_csr(o, c) as G:
                x, _ = G.pagerank(d, it)
                assert G.pagerank_windowed
                assert np.max(np.abs(x - xr) / xr) <= 1e-6
                x2, _ = G.pagerank(d, it, stealing=False)
                assert np.max(np.abs(x2 - xr) / xr) <= 1e-6
    # more than one target block of the far-arc bins (blocks of 2^22 vertices)
    big = sg.uk_like(n=5_000_000, seed=3, mu_ln=1.5, n_tendrils=10, tmin=20, tmax=40)
    xr = oracle.pagerank(big.off, big.col, 0.85, 5)
    with sage.load_csr(big.off, big.col) as G:
        x, _ = G.pagerank(0.85, 5)
        assert G.pagerank_windowed
        assert np.max(np.abs(x - xr) / xr) <= 1e-6
    # scrambled RMAT has no locality: the log-based push is kept
    g = sg.rmat(18, 16, seed=3, symmetric=False)
    with sage.load_csr(g.off, g.col) as G:
        x, _ = G.pagerank(0.85, 5)
        assert not G.pagerank_windowed


def test_outputs_in_place_and_translated(sage):
    """BFS levels / parents and SSSP distances written straight into caller device buffers (no
    output copy) equal the host-buffer path and the oracle — on the fused push path, the DO path,
    SSSP, and after a reorder (where the ids are translated and the in-place path is off); stale
    contents of the caller's buffer never leak through (the kernel initialises every entry)."""
    import torch
    g = sg.rmat(16, 16, seed=9, symmetric=True)
    w = sg.weights(g, 3)
    srcs = [int(x) for x in sg.sources(g, 3, seed=4)]
    with sage.load_csr(g.off, g.col, w, symmetric=True) as G:
        for rnd in range(2):
            for s in srcs:
                ref = oracle.bfs(g.off, g.col, s)
                for po in (True, False):
                    lv = torch.full((g.n,), 12345, dtype=torch.int32, device="cuda")
                    par = torch.full((g.n,), 777, dtype=torch.int32, device="cuda")
                    G.bfs(s, out=lv, parent_out=par, push_only=po)
                    lvh, parh, _ = G.bfs(s, parents=True, push_only=po)
                    assert np.array_equal(lv.cpu().numpy(), ref) and np.array_equal(lvh, ref)
                    _parents_ok(g.off, g.col, ref, par.cpu().numpy(), s)
                    _parents_ok(g.off, g.col, ref, parh, s)
                d = torch.full((g.n,), 5, dtype=torch.int32, device="cuda")
                G.sssp(s, out=d)
                dref, _ = oracle.sssp(g.off, g.col, w, s)
                assert np.array_equal(d.cpu().numpy().view(np.uint32), dref)
            if rnd == 0:
                G.reorder(rounds=1)


def test_pagerank_windowed_after_reorder(sage):
    """A reorder changes the labels, so the windowed push's locality is measured again; the ranks
    (original ids) stay equal to the oracle before and after."""
    uk = sg.uk_like(n=200000, seed=4, n_tendrils=10, tmin=20, tmax=60, hmax=1 << 12)
    xr = oracle.pagerank(uk.off, uk.col, 0.85, 10)
    with sage.load_csr(uk.off, uk.col) as G:
        x, _ = G.pagerank(0.85, 10)
        assert G.pagerank_windowed
        assert np.max(np.abs(x - xr) / xr) <= 1e-6
        G.reorder(rounds=1)
        x2, _ = G.pagerank(0.85, 10)
        assert np.max(np.abs(x2 - xr) / xr) <= 1e-6
