"""The CPU oracle for SAGE's hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product path (``libsage.so`` and its
binding ``paper_conf_sigmod_00020t21_b200``) never imports, links or executes anything here,
and nothing here imports the product: the two share no code.

The arithmetic lives in ``oracle.c`` (plain serial C, fp64 where floating point is involved);
this module only marshals numpy arrays.  Each wrapper names the paper passage it follows
(``P:NNN`` = line of the paper text).  Pins: ``tests/test_oracle_*.py``.
"""
from __future__ import annotations

import ctypes
import os
import sys

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None
OVERFLOW = 5


def _lib():
    global _LIB
    if _LIB is None:
        sys.path.insert(0, os.path.dirname(_HERE))
        from tools.build import build_oracle
        lib = ctypes.CDLL(build_oracle())
        i64, i32, dbl, p = ctypes.c_int64, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p
        lib.ora_bfs.argtypes = [i64, p, p, i32, p]
        lib.ora_check_bfs.argtypes = [i64, p, p, i32, p]
        lib.ora_sssp.argtypes = [i64, p, p, p, i32, p]
        lib.ora_check_sssp.argtypes = [i64, p, p, p, i32, p]
        lib.ora_pagerank.argtypes = [i64, p, p, dbl, i32, p]
        lib.ora_pagerank_step.argtypes = [i64, p, p, dbl, p, p]
        lib.ora_bc.argtypes = [i64, p, p, p, i64, p]
        lib.ora_tiles_row.argtypes = [i64, i64, i32, i32, i32, p]
        lib.ora_tiles_row.restype = i64
        lib.ora_tile_log.argtypes = [p, p, i64, i32, i32, i32, p]
        lib.ora_tile_log.restype = i64
        lib.ora_objective_tiles.argtypes = [i64, p, p, i32]
        lib.ora_objective_tiles.restype = i64
        lib.ora_sample_tiles.argtypes = [i64, p, p, i32, i32, i32, p, p, p]
        lib.ora_sample_tiles.restype = i64
        lib.ora_reorder_stages.argtypes = [i64, i64, p, p, i32, p, p, p, p, p, i32, p, p]
        lib.ora_reorder_match.argtypes = [i64, i32, p, p, p, p, p]
        lib.ora_reorder_match.restype = i64
        lib.ora_relabel.argtypes = [i64, p, p, p, p, p, p, p]
        _LIB = lib
    return _LIB


def _c(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a, a.ctypes.data


# ---------------------------------------------------------------- c1 BFS (Alg. 1 l.1-6)
def bfs(off, col, src: int) -> np.ndarray:
    """Hop levels from ``src`` (int32, -1 = unreachable): FIFO-queue BFS."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    n = len(off) - 1
    level = np.empty(n, dtype=np.int32)
    if _lib().ora_bfs(n, po, pc, int(src), level.ctypes.data) != 0:
        raise ValueError("bad source")
    return level


def check_bfs(off, col, src: int, level) -> int:
    """Certificate of SURVEY §8(c) c1; 0 = accepted."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    level, pl = _c(level, np.int32)
    return _lib().ora_check_bfs(len(off) - 1, po, pc, int(src), pl)


# ---------------------------------------------------------------- c2 SSSP (reading R4)
def sssp(off, col, w, src: int):
    """uint32 distances (UINT32_MAX = unreachable) by Dijkstra; returns (dist, overflow)."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    w, pw = _c(w, np.uint32)
    n = len(off) - 1
    dist = np.empty(n, dtype=np.uint32)
    rc = _lib().ora_sssp(n, po, pc, pw, int(src), dist.ctypes.data)
    if rc not in (0, OVERFLOW):
        raise ValueError("bad source")
    return dist, rc == OVERFLOW


def check_sssp(off, col, w, src: int, dist) -> int:
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    w, pw = _c(w, np.uint32)
    dist, pd = _c(dist, np.uint32)
    return _lib().ora_check_sssp(len(off) - 1, po, pc, pw, int(src), pd)


# ---------------------------------------------------------------- c3 PageRank (Alg. 1 l.26-29)
def pagerank(off, col, damping: float = 0.85, iters: int = 20) -> np.ndarray:
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    n = len(off) - 1
    x = np.empty(n, dtype=np.float64)
    if _lib().ora_pagerank(n, po, pc, float(damping), int(iters), x.ctypes.data) != 0:
        raise ValueError("empty graph")
    return x


def pagerank_step(off, col, x, damping: float = 0.85) -> np.ndarray:
    """One power-iteration step of c3 from the iterate ``x`` (same arithmetic as ``pagerank``)."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    x, px = _c(x, np.float64)
    n = len(off) - 1
    out = np.empty(n, dtype=np.float64)
    if _lib().ora_pagerank_step(n, po, pc, float(damping), px, out.ctypes.data) != 0:
        raise ValueError("empty graph")
    return out


# ---------------------------------------------------------------- BC (Alg. 1 l.8-24, NEXT #1)
def bc(off, col, sources) -> np.ndarray:
    """sum over s in ``sources`` of the Brandes dependencies delta_s(v) (v != s), fp64."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    src, ps = _c(np.atleast_1d(sources), np.int32)
    n = len(off) - 1
    out = np.empty(n, dtype=np.float64)
    if _lib().ora_bc(n, po, pc, ps, len(src), out.ctypes.data) != 0:
        raise ValueError("bad source")
    return out


# ---------------------------------------------------------------- c4 tiles (Alg. 2/3, Fig. 3)
def tiles_row(b: int, e: int, B: int = 256, M: int = 8, A: int = 4):
    """[(offset, size, kind)] for row [b, e); kind 0 = tile, 1 = fragment."""
    out = np.empty(3 * ((e - b) // B + 72), dtype=np.int64)
    k = _lib().ora_tiles_row(b, e, B, M, A, out.ctypes.data)
    return [tuple(int(x) for x in out[3 * i:3 * i + 3]) for i in range(k)]


def tile_log(off, vertices, B: int = 256, M: int = 8, A: int = 4) -> np.ndarray:
    """int64[k, 4] rows (vertex, offset, size, kind) of the resident tile log of ``vertices``."""
    off, po = _c(off, np.int64)
    vertices, pv = _c(vertices, np.int32)
    cap = 0
    deg = off[vertices.astype(np.int64) + 1] - off[vertices.astype(np.int64)]
    cap = int(np.sum(deg // B) + len(vertices) * 10 + 1)
    out = np.empty(4 * cap, dtype=np.int64)
    k = _lib().ora_tile_log(po, pv, len(vertices), B, M, A, out.ctypes.data)
    return out[:4 * k].reshape(k, 4)


# ---------------------------------------------------------------- §6 objective + c5 reorder
def sample_tiles(off, col, B: int = 256, M: int = 8, A: int = 4):
    """(tile_ptr int64[T+1], members int32[sum]) — every tile of every vertex (R19/R20)."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    n = len(off) - 1
    nm = ctypes.c_int64(0)
    nt = _lib().ora_sample_tiles(n, po, pc, B, M, A, None, None, ctypes.byref(nm))
    tile_ptr = np.empty(nt + 1, dtype=np.int64)
    members = np.empty(max(nm.value, 1), dtype=np.int32)
    _lib().ora_sample_tiles(n, po, pc, B, M, A, tile_ptr.ctypes.data, members.ctypes.data, None)
    return tile_ptr, members[:nm.value]


def objective_tiles(tile_ptr, members, S: int) -> int:
    """Σ_tiles count(distinct(floor(nbrs/S)))."""
    tile_ptr, pt = _c(tile_ptr, np.int64)
    members, pm = _c(members, np.int32)
    return int(_lib().ora_objective_tiles(len(tile_ptr) - 1, pt, pm, int(S)))


def objective(off, col, B: int = 256, M: int = 8, A: int = 4, S: int = 8) -> int:
    tp, mem = sample_tiles(off, col, B, M, A)
    return objective_tiles(tp, mem, S)


def reorder_stages(n: int, tile_ptr, members, S: int, candidates=None, trace_v: int = -1):
    """Stages 1-3 of one round.  Returns dict loc1, target, loc3, mover
    (+ "trace": [(lo, hi, L, R)] of each stage-2 step of vertex ``trace_v``)."""
    tile_ptr, pt = _c(tile_ptr, np.int64)
    members, pm = _c(members, np.int32)
    cand = None
    if candidates is not None:
        cm = np.zeros(n, dtype=np.uint8)
        cm[np.asarray(candidates, dtype=np.int64)] = 1
        cand = cm
    loc1, target, loc3 = (np.empty(n, dtype=np.int64) for _ in range(3))
    mover = np.empty(n, dtype=np.uint8)
    trace = np.zeros(4 * 64, dtype=np.int64)
    steps = ctypes.c_int32(0)
    _lib().ora_reorder_stages(n, len(tile_ptr) - 1, pt, pm, int(S),
                              cand.ctypes.data if cand is not None else None,
                              loc1.ctypes.data, target.ctypes.data, loc3.ctypes.data, mover.ctypes.data,
                              int(trace_v), trace.ctypes.data, ctypes.byref(steps))
    tr = [tuple(int(x) for x in trace[4 * k:4 * k + 4]) for k in range(steps.value)]
    return {"loc1": loc1, "target": target, "loc3": loc3, "mover": mover, "trace": tr}


def reorder_match(n: int, S: int, st) -> tuple[np.ndarray, int]:
    """Swap matching (R23) -> (sigma_round int32[n], #swaps)."""
    sig = np.empty(n, dtype=np.int32)
    loc1, target, loc3 = (np.ascontiguousarray(st[k], dtype=np.int64) for k in ("loc1", "target", "loc3"))
    mover = np.ascontiguousarray(st["mover"], dtype=np.uint8)
    swaps = _lib().ora_reorder_match(n, int(S), loc1.ctypes.data, target.ctypes.data, loc3.ctypes.data,
                                     mover.ctypes.data, sig.ctypes.data)
    return sig, int(swaps)


def relabel(off, col, w, sigma):
    """Row of sigma(v) = sort(sigma(adj v)), weights moved with their arcs (R24)."""
    off, po = _c(off, np.int64)
    col, pc = _c(col, np.int32)
    sigma, ps = _c(sigma, np.int32)
    n = len(off) - 1
    off2 = np.empty(n + 1, dtype=np.int64)
    col2 = np.empty(max(len(col), 1), dtype=np.int32)
    pw, w2, pw2 = None, None, None
    if w is not None:
        w, pw = _c(w, np.uint32)
        w2 = np.empty(max(len(w), 1), dtype=np.uint32)
        pw2 = w2.ctypes.data
    _lib().ora_relabel(n, po, pc, pw, ps, off2.ctypes.data, col2.ctypes.data, pw2)
    m = len(col)
    return off2, col2[:m], (w2[:m] if w2 is not None else None)


def reorder(off, col, w=None, rounds: int = 1, B: int = 256, M: int = 8, A: int = 4, S: int = 8,
            candidates=None):
    """``rounds`` rounds of Sampling-based Reordering ("round by round").

    Returns (off', col', w', sigma, per-round info) where sigma[v_orig] = current label.
    Stops early when a round has no movers (R25).  ``candidates`` (original IDs of the
    first round's labels) restricts movers, as in Figure 5's "only consider node-8".
    """
    off = np.ascontiguousarray(off, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    n = len(off) - 1
    sigma = np.arange(n, dtype=np.int32)
    info = []
    for r in range(rounds):
        tp, mem = sample_tiles(off, col, B, M, A)
        cand = None
        if candidates is not None:
            cand = sigma[np.asarray(candidates, dtype=np.int64)]
        st = reorder_stages(n, tp, mem, S, cand)
        nmov = int(st["mover"].sum())
        obj_before = objective_tiles(tp, mem, S)
        if nmov == 0:
            info.append({"movers": 0, "swaps": 0, "objective_before": obj_before})
            break
        sig_r, swaps = reorder_match(n, S, st)
        if swaps == 0:   # identity round: every later round would repeat it (R25)
            info.append({"movers": nmov, "swaps": 0, "objective_before": obj_before})
            break
        off, col, w = relabel(off, col, w, sig_r)
        sigma = sig_r[sigma]
        info.append({"movers": nmov, "swaps": swaps, "objective_before": obj_before})
    return off, col, w, sigma, info


# ---------------------------------------------------------------- online sampling (§6, NEXT #3)
def sample_tiles_weighted(off, col, weights, B: int = 256, M: int = 8, A: int = 4):
    """The tile sample of an ONLINE round ("the sampling is performed along with the tile
    access"; reading R19b): vertex u's tiles (kind 0, R20) occur weights[u] times — once per
    recorded access of u's row.  weights == 1 everywhere gives sample_tiles()."""
    col = np.ascontiguousarray(col, dtype=np.int32)
    verts = np.repeat(np.arange(len(off) - 1, dtype=np.int32), np.asarray(weights, dtype=np.int64))
    if len(verts) == 0:
        return np.zeros(1, dtype=np.int64), np.zeros(0, dtype=np.int32)
    q = tile_log(off, verts, B, M, A)
    q = q[q[:, 3] == 0]
    sizes = q[:, 2]
    tile_ptr = np.zeros(len(q) + 1, dtype=np.int64)
    np.cumsum(sizes, out=tile_ptr[1:])
    members = np.empty(int(tile_ptr[-1]), dtype=np.int32)
    for k, (_, o, s, _) in enumerate(q):          # plain copy of every occurrence's members
        members[tile_ptr[k]:tile_ptr[k] + s] = col[o:o + s]
    return tile_ptr, members


def reorder_round_weighted(off, col, w, weights, B: int = 256, M: int = 8, A: int = 4, S: int = 8):
    """One Sampling-based Reordering round (stages 1-3, swap matching, relabel; §6) over the
    weighted sample.  Returns (off', col', w', sigma_round, movers, swaps); sigma_round is the
    identity (and the graph unchanged) when there is no mover or no swap (R25)."""
    off = np.ascontiguousarray(off, dtype=np.int64)
    n = len(off) - 1
    tp, mem = sample_tiles_weighted(off, col, weights, B, M, A)
    st = reorder_stages(n, tp, mem, S)
    nmov = int(st["mover"].sum())
    ident = np.arange(n, dtype=np.int32)
    if nmov == 0:
        return off, col, w, ident, 0, 0
    sig_r, swaps = reorder_match(n, S, st)
    if swaps == 0:
        return off, col, w, ident, nmov, 0
    off2, col2, w2 = relabel(off, col, w, sig_r)
    return off2, col2, w2, sig_r, nmov, swaps


def online_reorder_bfs(off, col, sources, threshold=None, B: int = 256, M: int = 8, A: int = 4,
                       S: int = 8):
    """Online Sampling-based Reordering driven by a sequence of BFS queries (sage_online_reorder):
    every query records the rows of the vertices it reached (weight + 1 each, current labels); when
    the recorded row lengths since the last round reach ``threshold`` (default |E|), one
    round runs on that sample before the next query.  Returns (sigma, rounds, levels per query in
    original ids) with sigma[v_orig] = final label."""
    off = np.ascontiguousarray(off, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    n = len(off) - 1
    thr = len(col) if threshold is None or threshold <= 0 else int(threshold)
    sigma = np.arange(n, dtype=np.int32)
    weights = np.zeros(n, dtype=np.int64)
    acc, rounds, levels = 0, 0, []
    for s in sources:
        lv_cur = bfs(off, col, int(sigma[int(s)]))     # query in current labels
        levels.append(lv_cur[sigma])                   # answer in original ids
        reached = np.nonzero(lv_cur >= 0)[0]
        weights[reached] += 1
        acc += int(np.sum(off[reached + 1] - off[reached]))
        if acc >= thr:
            off, col, _, sig_r, _, _ = reorder_round_weighted(off, col, None, weights, B, M, A, S)
            sigma = sig_r[sigma]
            weights[:] = 0
            acc = 0
            rounds += 1
    return sigma, rounds, levels
