"""Seeded synthetic inputs (TEST / BENCH INFRASTRUCTURE — not the product, not the oracle).

Produces CSR graphs (``off`` int64[n+1], ``col`` int32[m]), integer weights and source
vertices from a counter-based hash, so every call with the same parameters returns the
same arrays on any machine and any thread count.  Holds none of SAGE's arithmetic; the
oracle (``oracle/``) and the CUDA path both consume what it returns.  The recipes are
SURVEY.md §8(d) (configs C1–C5) and are restated in DESIGN.md §"Input recipe".
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


class _CsrOut(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("m", ctypes.c_int64),
                ("off", ctypes.POINTER(ctypes.c_int64)), ("col", ctypes.POINTER(ctypes.c_int32))]


def _lib():
    global _LIB
    if _LIB is None:
        import sys
        sys.path.insert(0, os.path.dirname(_HERE))
        from tools.build import build_sagegen
        path = build_sagegen()
        lib = ctypes.CDLL(path)
        i64, u64, i32, dbl, p = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p
        lib.sg_rmat.argtypes = [ctypes.c_int, ctypes.c_int, u64, dbl, dbl, dbl, ctypes.c_int, ctypes.c_int,
                                ctypes.POINTER(_CsrOut)]
        lib.sg_twitter_like.argtypes = [i64, i64, u64, dbl, dbl, dbl, i64, i64, ctypes.POINTER(_CsrOut)]
        lib.sg_uk_like.argtypes = [i64, u64, dbl, dbl, i64, i64, dbl, dbl, dbl, i64, i64, i64,
                                   ctypes.POINTER(_CsrOut)]
        lib.sg_csr_from_tuples.argtypes = [i64, i64, p, p, ctypes.c_int, ctypes.POINTER(_CsrOut)]
        lib.sg_weights.argtypes = [i64, p, p, u64, ctypes.c_uint32, p]
        lib.sg_sources.argtypes = [i64, p, u64, i32, p]
        lib.sg_free.argtypes = [p]
        lib.sg_hash.argtypes = [u64, u64, u64]
        lib.sg_hash.restype = u64
        lib.sg_permute.argtypes = [u64, u64, u64]
        lib.sg_permute.restype = u64
        lib.sg_num_threads.restype = ctypes.c_int
        _LIB = lib
    return _LIB


@dataclass
class Graph:
    """A host CSR graph: rows sorted ascending, no self loops, no duplicate arcs."""
    n: int
    off: np.ndarray          # int64[n+1]
    col: np.ndarray          # int32[m]
    symmetric: bool
    name: str = ""
    w: np.ndarray | None = None   # uint32[m] or None

    @property
    def m(self) -> int:
        return int(self.off[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.off)


def _take(out: _CsrOut, symmetric: bool, name: str) -> Graph:
    n, m = out.n, out.m
    lib = _lib()
    off = np.ctypeslib.as_array(out.off, shape=(n + 1,)).copy()
    col = np.ctypeslib.as_array(out.col, shape=(max(m, 1),))[:m].copy()
    lib.sg_free(ctypes.cast(out.off, ctypes.c_void_p))
    lib.sg_free(ctypes.cast(out.col, ctypes.c_void_p))
    return Graph(n=n, off=off, col=col, symmetric=symmetric, name=name)


def rmat(scale: int, edgefactor: int = 16, seed: int = 1, symmetric: bool = True,
         scramble: bool = True, abc=(0.57, 0.19, 0.19)) -> Graph:
    """Graph500 Kronecker/RMAT: 2^scale vertices, edgefactor·2^scale tuples."""
    out = _CsrOut()
    rc = _lib().sg_rmat(scale, edgefactor, seed, abc[0], abc[1], abc[2], int(symmetric), int(scramble),
                        ctypes.byref(out))
    if rc != 0:
        raise ValueError("sg_rmat failed")
    return _take(out, symmetric, f"rmat{scale}{'s' if symmetric else 'd'}_ef{edgefactor}_seed{seed}")


def twitter_like(n: int = 41_600_000, tuples: int = 1_590_000_000, seed: int = 1, s_out: float = 0.72,
                 s_in: float = 0.65, mu: float = 0.5, cmin: int = 32, cmax: int = 65536) -> Graph:
    """Directed power-law social graph shaped like twitter (Table 1).
    Tuple count tuned so that the kept arcs are ~1.46e9 (round 1 kept 1.38e9 of 1.5e9 tuples)."""
    out = _CsrOut()
    rc = _lib().sg_twitter_like(n, tuples, seed, s_out, s_in, mu, cmin, cmax, ctypes.byref(out))
    if rc != 0:
        raise ValueError("sg_twitter_like failed")
    return _take(out, False, f"twitter_like_n{n}_t{tuples}_seed{seed}")


def uk_like(n: int = 105_000_000, seed: int = 1, mu_ln: float = 3.40, sigma_ln: float = 1.1,
            dmax: int = 10_000, hmax: int = 1 << 20, p_local: float = 0.8, goff: float = 16.0,
            s_glob: float = 0.8, n_tendrils: int = 2000, tmin: int = 50, tmax: int = 500) -> Graph:
    """Directed high-diameter web graph in crawl order.  mu_ln = 3.40 keeps
    ~35.1 arcs per vertex after duplicate removal (~3.7e9 arcs at n = 105M; measured 33.8 / 36.5
    at mu_ln 3.35 / 3.45 on n = 4M)."""
    out = _CsrOut()
    rc = _lib().sg_uk_like(n, seed, mu_ln, sigma_ln, dmax, hmax, p_local, goff, s_glob, n_tendrils,
                           tmin, tmax, ctypes.byref(out))
    if rc != 0:
        raise ValueError("sg_uk_like failed")
    return _take(out, False, f"uk_like_n{n}_seed{seed}")


def from_edges(n: int, edges, symmetric: bool = False, name: str = "edges") -> Graph:
    """CSR from an explicit (u, v) list: self loops and duplicates dropped, rows sorted."""
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    src = np.ascontiguousarray(e[:, 0].astype(np.int32))
    dst = np.ascontiguousarray(e[:, 1].astype(np.int32))
    out = _CsrOut()
    rc = _lib().sg_csr_from_tuples(n, len(src), src.ctypes.data, dst.ctypes.data, int(symmetric),
                                   ctypes.byref(out))
    if rc != 0:
        raise ValueError("vertex id out of range")
    return _take(out, symmetric, name)


def random_graph(n: int, m_tuples: int, seed: int, symmetric: bool = False) -> Graph:
    """Uniform random tuples (for brute-force pins on tiny graphs)."""
    lib = _lib()
    src = np.array([lib.sg_hash(seed, i, 0) % n for i in range(m_tuples)], dtype=np.int64)
    dst = np.array([lib.sg_hash(seed, i, 1) % n for i in range(m_tuples)], dtype=np.int64)
    return from_edges(n, np.stack([src, dst], 1), symmetric, f"rand_n{n}_t{m_tuples}_seed{seed}")


def weights(g: Graph, seed: int = 1, wmax: int = 255) -> np.ndarray:
    """Symmetric uint32 weights in [1, wmax]: w(u,v) = 1 + hash(seed, min, max) mod wmax (R4)."""
    w = np.empty(g.m, dtype=np.uint32)
    _lib().sg_weights(g.n, g.off.ctypes.data, g.col.ctypes.data, seed, wmax, w.ctypes.data)
    return w


def sources(g: Graph, k: int, seed: int = 2) -> np.ndarray:
    """k seeded sources, uniform over vertices with out-degree > 0 (R29)."""
    out = np.empty(k, dtype=np.int32)
    if _lib().sg_sources(g.n, g.off.ctypes.data, seed, k, out.ctypes.data) != 0:
        raise ValueError("graph has no vertex with out-degree > 0")
    return out


def num_threads() -> int:
    return _lib().sg_num_threads()


def config(name: str) -> Graph:
    """The named workloads of BASELINE.json / SURVEY §8.0 (weights attached where the config uses them)."""
    if name == "C1":
        return rmat(16, 16, 1, True)
    if name == "C2":
        g = rmat(24, 16, 1, True)
        g.w = weights(g, 1)
        return g
    if name == "C3":
        return twitter_like()
    if name == "C4":
        return uk_like()
    raise KeyError(name)


# ---------------------------------------------------------------- per-rank device generation
_DEV = None


def _dev_lib():
    global _DEV
    if _DEV is None:
        import sys
        sys.path.insert(0, os.path.dirname(_HERE))
        from tools.build import build_sagegen_dev
        lib = ctypes.CDLL(build_sagegen_dev())
        i64, u64, p, dbl, c_int = ctypes.c_longlong, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_double, ctypes.c_int
        lib.sgd_rmat_build.argtypes = [c_int, c_int, u64, dbl, dbl, dbl, c_int, i64, i64, p,
                                       ctypes.POINTER(p), ctypes.POINTER(i64)]
        lib.sgd_rmat_take.argtypes = [p, p, p, p]
        lib.sgd_weights.argtypes = [i64, i64, p, p, u64, ctypes.c_uint32, p, p]
        lib.sgd_free.argtypes = [p]
        _DEV = lib
    return _DEV


def rmat_device(scale: int, edgefactor: int = 16, seed: int = 1, symmetric: bool = True,
                v_begin: int = 0, v_end: int | None = None, weights_seed: int | None = None,
                abc=(0.57, 0.19, 0.19), stream=None):
    """Rows [v_begin, v_end) of ``rmat(scale, edgefactor, seed, symmetric)`` generated on the current
    CUDA device (every tuple is regenerated; arcs whose source is outside the block are dropped).
    Returns torch tensors (off int64[n_local+1] rebased to 0, col int32[m_local], w uint32 or None)."""
    import torch
    n = 1 << scale
    v_end = n if v_end is None else v_end
    st = torch.cuda.current_stream().cuda_stream if stream is None else stream
    h, m = ctypes.c_void_p(), ctypes.c_longlong(0)
    rc = _dev_lib().sgd_rmat_build(scale, edgefactor, seed, abc[0], abc[1], abc[2], int(symmetric), v_begin, v_end,
                                   st, ctypes.byref(h), ctypes.byref(m))
    if rc != 0:
        raise RuntimeError(f"sgd_rmat_build failed ({rc})")
    off = torch.empty(v_end - v_begin + 1, dtype=torch.int64, device="cuda")
    col = torch.empty(max(m.value, 1), dtype=torch.int32, device="cuda")
    if _dev_lib().sgd_rmat_take(h, off.data_ptr(), col.data_ptr(), st) != 0:
        raise RuntimeError("sgd_rmat_take failed")
    col = col[:m.value]
    w = None
    if weights_seed is not None:
        w = torch.empty(max(m.value, 1), dtype=torch.int32, device="cuda").view(torch.uint32)
        if _dev_lib().sgd_weights(v_end - v_begin, v_begin, off.data_ptr(), col.data_ptr(), weights_seed, 255,
                                  w.data_ptr(), st) != 0:
            raise RuntimeError("sgd_weights failed")
        w = w[:m.value]
    return off, col, w


def hash3(seed: int, a: int, b: int) -> int:
    """The generators' counter-based hash (splitmix64 of (seed, a, b)); sources use (seed, i, try)."""
    return int(_lib().sg_hash(seed, a, b))
