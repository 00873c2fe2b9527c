"""Pins for the tile-decomposition (c4) and Sampling-based Reordering (c5) oracles.

* Figure 3 worked example — golden fixture tests/golden/fig3_tiles.json,
* decomposition invariants on random rows,
* Figure 5 worked example — golden fixture tests/golden/fig5_reorder.json:
  stage-1 vector, node-8's stage-2 counts, its stage-3 locality, the 8<->3 swap and the
  sorted 2nd-round tiles, the objective before/after,
* the objective on Theorem 6.1's tile<2> special case vs its MLA-with-binary-
  distancing form, brute-forced over all permutations,
* invariants of a full reorder round: sigma is a bijection, the relabelled CSR is isomorphic,
  BFS/SSSP/PR answers are unchanged in original IDs.
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
import sagegen as sg


def test_figure3(golden_dir):
    fx = json.load(open(os.path.join(golden_dir, "fig3_tiles.json")))
    for row in fx["rows"]:
        got = oracle.tiles_row(row["begin"], row["end"], fx["B"], fx["M"], fx["A"])
        assert got == [tuple(t) for t in row["tiles"]], row["color"]


@pytest.mark.parametrize("B,M,A", [(256, 8, 0), (256, 8, 4), (256, 8, 32), (1024, 32, 4), (16, 8, 0)])
def test_decomposition_invariants(B, M, A):
    rng = np.random.default_rng(B + M + A)
    for _ in range(3000):
        b = int(rng.integers(0, 10**6))
        d = int(rng.choice([0, 1, 3, 7, 8, 9, 31, 255, 256, 257, 1000, 5000, 70000]))
        d = max(0, d + int(rng.integers(-2, 3)))
        e = b + d
        ts = oracle.tiles_row(b, e, B, M, A)
        pos = b
        sub = set()
        for k, (o, s, kind) in enumerate(ts):
            assert o == pos and s > 0
            pos += s
            if kind == 0:
                assert s in [B >> i for i in range(0, 20) if (B >> i) >= M]
                if A:
                    assert o % min(A, s) == 0  # aligned tiles (R14)
                if s < B:
                    assert s not in sub
                    sub.add(s)
            else:
                # fragments: an aligned head (< A) and/or a tail (< M)
                assert (k == 0 and A and s < A) or (k == len(ts) - 1 and s < M)
        assert pos == e


def _fig5_csr(fx):
    """A CSR whose tile sample (B = M = 4, A = 0) is exactly Figure 5's four tiles.
    Rows are owned by vertices 6, 7, 11, 13, which appear in no tile."""
    owners = [6, 7, 11, 13]
    edges = [(o, v) for o, t in zip(owners, fx["tiles"]) for v in t]
    return sg.from_edges(fx["n"], edges)


def test_figure5_stages(golden_dir):
    fx = json.load(open(os.path.join(golden_dir, "fig5_reorder.json")))
    g = _fig5_csr(fx)
    tp, mem = oracle.sample_tiles(g.off, g.col, B=4, M=4, A=0)
    assert [sorted(mem[tp[i]:tp[i + 1]].tolist()) for i in range(len(tp) - 1)] == fx["tiles"]
    st = oracle.reorder_stages(g.n, tp, mem, fx["S"], candidates=[8], trace_v=8)
    assert st["loc1"].tolist() == fx["stage1_locality"]
    assert [(lo, hi, L, R) for lo, hi, L, R in st["trace"]] == \
        [(s["lo"], s["hi"], s["left"], s["right"]) for s in fx["node8_stage2"]]
    assert st["target"][8] == fx["node8_target_sector"]
    assert st["loc3"][8] == fx["node8_loc3"]
    assert st["mover"].nonzero()[0].tolist() == [8]
    assert oracle.objective_tiles(tp, mem, fx["S"]) == fx["objective_round1"]


def test_figure5_node8_round(golden_dir):
    fx = json.load(open(os.path.join(golden_dir, "fig5_reorder.json")))
    g = _fig5_csr(fx)
    off2, col2, _, sigma, info = oracle.reorder(g.off, g.col, None, rounds=1, B=4, M=4, A=0, S=fx["S"],
                                                candidates=[8])
    assert sigma[8] == fx["node8_only_new_label"] and sigma[3] == 8
    assert info[0]["swaps"] == 1
    tp, mem = oracle.sample_tiles(off2, col2, B=4, M=4, A=0)
    tiles = sorted(mem[tp[i]:tp[i + 1]].tolist() for i in range(len(tp) - 1))
    assert tiles == sorted(fx["round2_tiles_node8_only"])
    assert oracle.objective_tiles(tp, mem, fx["S"]) == fx["objective_round2_node8_only"]


def test_figure5_full_run_reading(golden_dir):
    fx = json.load(open(os.path.join(golden_dir, "fig5_reorder.json")))
    exp = fx["reading_full_run"]
    g = _fig5_csr(fx)
    tp, mem = oracle.sample_tiles(g.off, g.col, B=4, M=4, A=0)
    st = oracle.reorder_stages(g.n, tp, mem, fx["S"])
    assert st["mover"].nonzero()[0].tolist() == exp["movers"]
    sig, swaps = oracle.reorder_match(g.n, fx["S"], st)
    pairs = sorted(tuple(sorted((v, int(sig[v])))) for v in range(g.n) if sig[v] != v)
    assert sorted(set(pairs)) == [tuple(p) for p in exp["swaps"]] and swaps == len(exp["swaps"])
    off2, col2, _ = oracle.relabel(g.off, g.col, None, sig)
    assert oracle.objective(off2, col2, B=4, M=4, A=0, S=fx["S"]) == exp["objective_after"]


def test_objective_theorem61_special_case():
    """tile<2> per edge: objective = |E| + #edges whose ends fall in different sectors,
    i.e. |E| + sum f(|sigma u - sigma v|) with binary distancing only when sectors are aligned.
    Brute force over all permutations of n = 6 checks the objective function itself."""
    n, S = 6, 2
    edges = [(0, 3), (1, 4), (2, 5), (0, 5), (3, 4)]
    best = None
    for perm in itertools.permutations(range(n)):
        members = np.array([perm[x] for e in edges for x in e], dtype=np.int32)
        tp = np.arange(0, 2 * len(edges) + 1, 2, dtype=np.int64)
        obj = oracle.objective_tiles(tp, members, S)
        cross = sum(1 for u, v in edges if perm[u] // S != perm[v] // S)
        assert obj == len(edges) + cross
        best = obj if best is None else min(best, obj)
    # a perfect matching of 3 sector pairs can internalise at most 3 of the 5 edges
    assert best == len(edges) + 2


def _canon(off, col, w):
    return sorted((u, int(c), int(w[k]) if w is not None else 0)
                  for u in range(len(off) - 1) for k, c in enumerate(col[off[u]:off[u + 1]], start=off[u]))


@pytest.mark.parametrize("sym", [True, False])
def test_reorder_invariants(sym):
    g = sg.rmat(10, 16, seed=11, symmetric=sym)
    w = sg.weights(g, 3)
    off2, col2, w2, sigma, info = oracle.reorder(g.off, g.col, w, rounds=3, B=32, M=8, A=4, S=8)
    n = g.n
    assert sorted(sigma.tolist()) == list(range(n))             # bijection
    assert all(np.all(np.diff(col2[off2[u]:off2[u + 1]]) > 0) for u in range(n))   # sorted rows
    # isomorphic: relabelled arcs = sigma(original arcs), weights carried along
    src = np.repeat(np.arange(n), np.diff(g.off))
    orig = sorted(zip(sigma[src].tolist(), sigma[g.col].tolist(), w.tolist()))
    src2 = np.repeat(np.arange(n), np.diff(off2))
    assert orig == sorted(zip(src2.tolist(), col2.tolist(), w2.tolist()))
    assert info[0]["movers"] > 0
    # query answers unchanged in original IDs
    for s in sg.sources(g, 3):
        s = int(s)
        assert np.array_equal(oracle.bfs(off2, col2, int(sigma[s]))[sigma], oracle.bfs(g.off, g.col, s))
        d1, _ = oracle.sssp(off2, col2, w2, int(sigma[s]))
        d0, _ = oracle.sssp(g.off, g.col, w, s)
        assert np.array_equal(d1[sigma], d0)
    x0 = oracle.pagerank(g.off, g.col)
    x1 = oracle.pagerank(off2, col2)[sigma]
    assert np.max(np.abs(x1 - x0) / x0) < 1e-12


def test_reorder_improves_objective_on_scrambled_rmat():
    g = sg.rmat(11, 16, seed=1, symmetric=True)
    before = oracle.objective(g.off, g.col, B=256, M=8, A=4, S=8)
    off2, col2, _, _, info = oracle.reorder(g.off, g.col, None, rounds=2, B=256, M=8, A=4, S=8)
    after = oracle.objective(off2, col2, B=256, M=8, A=4, S=8)
    assert info[0]["swaps"] > 0 and after < before


def test_tile_log_quads_with_fragments(golden_dir):
    """Hand-derived resident tile log quadruples (vertex, offset, size, kind) with aligned head
    fragments, tail fragments, empty rows and several ladders (tests/golden/tile_log_quads.json)."""
    fx = json.load(open(os.path.join(golden_dir, "tile_log_quads.json")))
    off = np.array(fx["off"], dtype=np.int64)
    vs = np.array(fx["vertices"], dtype=np.int32)
    for lad in fx["ladders"]:
        got = oracle.tile_log(off, vs, lad["B"], lad["M"], lad["A"]).tolist()
        assert got == lad["quads"], (lad["B"], lad["M"], lad["A"])


def _tie_csr(fx):
    n = fx["n"]
    rows = {int(k): v for k, v in fx["rows"].items()}
    off = np.zeros(n + 1, dtype=np.int64)
    for u in range(n):
        off[u + 1] = off[u] + len(rows.get(u, []))
    col = np.array([c for u in range(n) for c in rows.get(u, [])], dtype=np.int32)
    return off, col


def test_stage2_tie_goes_left(golden_dir):
    """Reading R21's tie rule (L == R -> left half) on a hand-built sample whose first stage-2
    step ties (tests/golden/stage2_tie.json)."""
    fx = json.load(open(os.path.join(golden_dir, "stage2_tie.json")))
    off, col = _tie_csr(fx)
    tp, mem = oracle.sample_tiles(off, col, fx["B"], fx["M"], fx["A"])
    st = oracle.reorder_stages(fx["n"], tp, mem, fx["S"], trace_v=1)
    assert [list(t) for t in st["trace"]] == fx["trace_v1"]
    assert st["target"][1] == fx["target_v1"]
    assert st["loc1"][1] == fx["loc1_v1"] and st["loc3"][1] == fx["loc3_v1"]
    assert st["mover"][1] == fx["mover_v1"]
