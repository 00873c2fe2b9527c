"""Python binding of libsage.so — the B200-native SAGE hot path (argument marshalling only).

Every step of BFS / SSSP / PageRank / reordering runs in the CUDA kernels of ``csrc/`` behind
the C ABI of ``include/sage.h``; this module only converts arrays to pointers.  There is no CPU
fallback: if the extension is missing or there is no GPU, calls raise ``SageError``.

Names follow the C ABI: ``load_csr`` -> ``sage_load_csr``, ``Graph.bfs`` -> ``sage_bfs_ex`` …
Arrays may be numpy arrays (host) or torch tensors (host or CUDA); outputs default to numpy.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, os.environ.get("SAGE_LIB", "libsage.so"))

OK, E_INVALID, E_NOMEM, E_CUDA, E_NCCL, E_OVERFLOW, E_UNSUPPORTED = range(7)
F_SYMMETRIC, F_DEVICE_PTRS, F_BORROW, F_NO_VALIDATE, F_PUSH_ONLY, F_NO_STEALING = 1, 2, 4, 8, 16, 64
F_HOST_COLUMNS = 128
STATUS_NAMES = {0: "SAGE_OK", 1: "SAGE_E_INVALID", 2: "SAGE_E_NOMEM", 3: "SAGE_E_CUDA",
                4: "SAGE_E_NCCL", 5: "SAGE_E_OVERFLOW", 6: "SAGE_E_UNSUPPORTED"}

EXPORTED = ["sage_load_csr", "sage_free", "sage_bfs", "sage_bfs_ex", "sage_sssp", "sage_pagerank",
            "sage_pagerank_ex", "sage_bc", "sage_online_reorder", "sage_online_reorder_info",
            "sage_reorder", "sage_reorder_objective", "sage_get_permutation", "sage_get_csr", "sage_graph_info",
            "sage_debug_export_tiles", "sage_debug_reorder_stages", "sage_nccl_unique_id", "sage_debug_level_records", "sage_debug_loopback_id", "sage_last_error", "sage_version"]


class SageError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class Options(ctypes.Structure):
    _fields_ = [("tile_cta", ctypes.c_int32), ("tile_min", ctypes.c_int32), ("align", ctypes.c_int32),
                ("alpha", ctypes.c_double), ("beta", ctypes.c_double), ("ctas_per_sm", ctypes.c_int32),
                ("hub_filter", ctypes.c_int32)]


class Dist(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("nccl_unique_id", ctypes.c_void_p),
                ("v_begin", ctypes.c_int64), ("v_end", ctypes.c_int64), ("exchange", ctypes.c_int32)]


class Csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("m", ctypes.c_int64), ("row_offsets", ctypes.c_void_p),
                ("col_indices", ctypes.c_void_p), ("weights", ctypes.c_void_p), ("flags", ctypes.c_uint32),
                ("cuda_stream", ctypes.c_void_p), ("opts", ctypes.POINTER(Options)),
                ("dist", ctypes.POINTER(Dist))]


class Stats(ctypes.Structure):
    _fields_ = [("levels", ctypes.c_int32), ("push_levels", ctypes.c_int32), ("pull_levels", ctypes.c_int32),
                ("edges_traversed", ctypes.c_int64), ("arcs_inspected", ctypes.c_int64),
                ("vertices_expanded", ctypes.c_int64), ("vertices_discovered", ctypes.c_int64),
                ("ms", ctypes.c_double), ("model_bytes", ctypes.c_double), ("kernel_ms", ctypes.c_double)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class ReorderOpts(ctypes.Structure):
    _fields_ = [("sector_width", ctypes.c_int32), ("candidates", ctypes.c_void_p),
                ("n_candidates", ctypes.c_int64)]


_LIB = None


def lib():
    """Load libsage.so (raises if it is missing: no fallback)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing; build it with `python -c 'import __graft_entry__ as g; "
                              f"g.build()'` (nvcc, sm_100a)")
        L = ctypes.CDLL(LIB_PATH)
        p, i32, i64, u32, dbl = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_double
        L.sage_load_csr.argtypes = [ctypes.POINTER(Csr), ctypes.POINTER(p)]
        L.sage_free.argtypes = [p]
        L.sage_bfs.argtypes = [p, i32, p, p, ctypes.POINTER(Stats)]
        L.sage_online_reorder.argtypes = [p, i32, i32, i64]
        L.sage_online_reorder_info.argtypes = [p, ctypes.POINTER(i64), ctypes.POINTER(i64), ctypes.POINTER(i64)]
        L.sage_bfs_ex.argtypes = [p, i32, p, p, u32, ctypes.POINTER(Stats)]
        L.sage_sssp.argtypes = [p, i32, p, ctypes.POINTER(Stats)]
        L.sage_pagerank.argtypes = [p, dbl, i32, p, ctypes.POINTER(Stats)]
        L.sage_pagerank_ex.argtypes = [p, dbl, i32, p, u32, ctypes.POINTER(Stats)]
        L.sage_bc.argtypes = [p, p, i64, p, ctypes.POINTER(Stats)]
        L.sage_reorder.argtypes = [p, i32, ctypes.POINTER(ReorderOpts), ctypes.POINTER(Stats)]
        L.sage_get_permutation.argtypes = [p, p]
        L.sage_reorder_objective.argtypes = [p, i32, p]
        L.sage_debug_reorder_stages.argtypes = [p, i32, p, i64, p, p, p, p]
        L.sage_get_csr.argtypes = [p, p, p, p]
        L.sage_graph_info.argtypes = [p, p, p, p, p, p]
        L.sage_debug_export_tiles.argtypes = [p, p, i64, p, i64, p]
        L.sage_debug_level_records.argtypes = [p, p, i32, p]
        L.sage_nccl_unique_id.argtypes = [p]
        L.sage_debug_loopback_id.argtypes = [i32, p]
        L.sage_last_error.restype = ctypes.c_char_p
        L.sage_version.restype = ctypes.c_char_p
        for f in EXPORTED:
            if f not in ("sage_last_error", "sage_version"):
                getattr(L, f).restype = ctypes.c_int
        _LIB = L
    return _LIB


def last_error() -> str:
    return lib().sage_last_error().decode()


def version() -> str:
    return lib().sage_version().decode()


def _check(status: int):
    if status != OK:
        raise SageError(status, last_error())


def _is_torch(a) -> bool:
    return type(a).__module__.startswith("torch")


def _ptr(a, dtype):
    """(pointer, keepalive, is_device) of a numpy array / torch tensor with the given numpy dtype."""
    if a is None:
        return None, None, False
    if _is_torch(a):
        import torch
        tdt = {np.int64: torch.int64, np.int32: torch.int32, np.uint32: torch.uint32,
               np.float64: torch.float64}[np.dtype(dtype).type]
        if a.dtype != tdt or not a.is_contiguous():
            raise TypeError(f"tensor must be contiguous {tdt}, got {a.dtype}")
        return a.data_ptr(), a, a.is_cuda
    arr = np.ascontiguousarray(a, dtype=dtype)
    return arr.ctypes.data, arr, False


@dataclass
class _Out:
    ptr: int
    obj: object


def _out(out, n, dtype):
    if out is None:
        arr = np.empty(n, dtype=dtype)
        return _Out(arr.ctypes.data, arr)
    if _is_torch(out):
        return _Out(out.data_ptr(), out)
    if not (isinstance(out, np.ndarray) and out.flags.c_contiguous and out.dtype == dtype and out.size >= n):
        raise TypeError("out must be a contiguous array of the right dtype and size")
    return _Out(out.ctypes.data, out)


class Graph:
    """A device-resident CSR graph (opaque ``sage_graph``)."""

    def __init__(self, handle: int, keep):
        self._h = ctypes.c_void_p(handle)
        self._keep = keep          # borrowed arrays stay alive as long as the graph
        n, m, nl, vb, fl = (ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(),
                            ctypes.c_uint32())
        _check(lib().sage_graph_info(self._h, ctypes.byref(n), ctypes.byref(m), ctypes.byref(nl),
                                     ctypes.byref(vb), ctypes.byref(fl)))
        self.n, self.m, self.n_local, self.v_begin, self.flags = n.value, m.value, nl.value, vb.value, fl.value

    @property
    def handle(self):
        return self._h

    @property
    def peer_exchange(self) -> bool:
        """Multi-GPU: the push frontier exchange runs over peer memory (sage_dist.exchange = 0)."""
        return bool(self.flags & 0x400)

    @property
    def pagerank_windowed(self) -> bool:
        """Push PageRank runs the windowed form (chosen at the first push PageRank call)."""
        fl = ctypes.c_uint32()
        _check(lib().sage_graph_info(self._h, None, None, None, None, ctypes.byref(fl)))
        return bool(fl.value & 0x800)

    def free(self):
        if self._h:
            lib().sage_free(self._h)
            self._h = ctypes.c_void_p(0)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.free()

    @property
    def rows_sorted(self) -> bool:
        return bool(self.flags & 0x100)

    # ------------------------------------------------------------------ queries
    def bfs(self, source: int, out=None, parent_out=None, parents: bool = False, push_only: bool = False,
            stealing: bool = True):
        """sage_bfs_ex -> (level int32[n_local], parent or None, stats dict)."""
        o = _out(out, self.n_local, np.int32)
        po = None
        if parents or parent_out is not None:
            po = _out(parent_out, self.n_local, np.int32)
        st = Stats()
        fl = (F_PUSH_ONLY if push_only else 0) | (0 if stealing else F_NO_STEALING)
        _check(lib().sage_bfs_ex(self._h, int(source), o.ptr, po.ptr if po else None, fl, ctypes.byref(st)))
        return o.obj, (po.obj if po else None), st.as_dict()

    def sssp(self, source: int, out=None):
        o = _out(out, self.n_local, np.uint32)
        st = Stats()
        _check(lib().sage_sssp(self._h, int(source), o.ptr, ctypes.byref(st)))
        return o.obj, st.as_dict()

    def pagerank(self, damping: float = 0.85, iterations: int = 20, out=None, push_only: bool = False,
                 stealing: bool = True):
        """sage_pagerank_ex (pull form on symmetric graphs unless push_only; stealing=False runs the
        log-based push without stealing, never the windowed form)."""
        o = _out(out, self.n_local, np.float64)
        st = Stats()
        fl = (F_PUSH_ONLY if push_only else 0) | (0 if stealing else F_NO_STEALING)
        _check(lib().sage_pagerank_ex(self._h, float(damping), int(iterations), o.ptr, fl, ctypes.byref(st)))
        return o.obj, st.as_dict()

    def bc(self, sources, out=None):
        """sage_bc: sum over ``sources`` of the Brandes dependencies (fp64)."""
        src = np.ascontiguousarray(np.atleast_1d(sources), dtype=np.int32)
        o = _out(out, self.n_local, np.float64)
        st = Stats()
        _check(lib().sage_bc(self._h, src.ctypes.data, len(src), o.ptr, ctypes.byref(st)))
        return o.obj, st.as_dict()

    def online_reorder(self, enable: bool = True, sector_width: int = 8, threshold: int = 0):
        """sage_online_reorder: record the tile accesses of later queries; one reorder round each
        time the recorded row lengths reach ``threshold`` (0 = |E|)."""
        _check(lib().sage_online_reorder(self._h, 1 if enable else 0, int(sector_width), int(threshold)))

    def online_info(self) -> dict:
        """sage_online_reorder_info -> {"rounds", "swaps", "pending"}."""
        r, s, p = ctypes.c_int64(0), ctypes.c_int64(0), ctypes.c_int64(0)
        _check(lib().sage_online_reorder_info(self._h, ctypes.byref(r), ctypes.byref(s), ctypes.byref(p)))
        return {"rounds": r.value, "swaps": s.value, "pending": p.value}

    def reorder(self, rounds: int = 1, sector_width: int = 8, candidates=None):
        ro = ReorderOpts()
        ro.sector_width = sector_width
        keep = None
        if candidates is not None:
            keep = np.ascontiguousarray(candidates, dtype=np.int32)
            ro.candidates = keep.ctypes.data
            ro.n_candidates = len(keep)
        st = Stats()
        _check(lib().sage_reorder(self._h, int(rounds), ctypes.byref(ro), ctypes.byref(st)))
        return st.as_dict()

    def objective(self, sector_width: int = 8) -> int:
        """sage_reorder_objective: sum over sampled tiles of distinct sectors."""
        out = ctypes.c_int64(0)
        _check(lib().sage_reorder_objective(self._h, int(sector_width), ctypes.byref(out)))
        return out.value

    def reorder_stages(self, sector_width: int = 8, candidates=None) -> dict:
        """sage_debug_reorder_stages -> {loc1, target, loc3, mover} of one round (no relabel)."""
        n = self.n
        out = {k: np.zeros(n, dtype=np.int64) for k in ("loc1", "target", "loc3")}
        mover = np.zeros(n, dtype=np.uint8)
        c = None if candidates is None else np.ascontiguousarray(candidates, dtype=np.int32)
        _check(lib().sage_debug_reorder_stages(self._h, int(sector_width), c.ctypes.data if c is not None else None,
                                               0 if c is None else len(c), out["loc1"].ctypes.data,
                                               out["target"].ctypes.data, out["loc3"].ctypes.data,
                                               mover.ctypes.data))
        out["mover"] = mover
        return out

    def permutation(self) -> np.ndarray:
        out = np.empty(self.n, dtype=np.int32)
        _check(lib().sage_get_permutation(self._h, out.ctypes.data))
        return out

    def csr(self):
        off = np.empty(self.n_local + 1, dtype=np.int64)
        col = np.empty(max(self.m, 1), dtype=np.int32)
        w = np.empty(max(self.m, 1), dtype=np.uint32)
        _check(lib().sage_get_csr(self._h, off.ctypes.data, col.ctypes.data, w.ctypes.data))
        return off, col[:self.m], w[:self.m]

    def level_records(self) -> np.ndarray:
        """sage_debug_level_records -> int64[levels, 9] (dir, |F|, arcs(F), inspected, scanned,
        discovered, t_ns at level end, t_ns when the last warp finished, t_ns at the end of the
        expansion phase) of the last BFS/SSSP query."""
        n = ctypes.c_int32(0)
        buf = np.zeros(9 * 4096, dtype=np.int64)
        _check(lib().sage_debug_level_records(self._h, buf.ctypes.data, 4096, ctypes.byref(n)))
        return buf[:9 * min(n.value, 4096)].reshape(-1, 9)

    def export_tiles(self, vertices) -> np.ndarray:
        """sage_debug_export_tiles -> int64[k, 4] (vertex, offset, size, kind)."""
        v = np.ascontiguousarray(vertices, dtype=np.int32)
        nq = ctypes.c_int64(0)
        _check(lib().sage_debug_export_tiles(self._h, v.ctypes.data, len(v), None, 0, ctypes.byref(nq)))
        out = np.empty(4 * max(nq.value, 1), dtype=np.int64)
        _check(lib().sage_debug_export_tiles(self._h, v.ctypes.data, len(v), out.ctypes.data, nq.value,
                                             ctypes.byref(nq)))
        return out[:4 * nq.value].reshape(-1, 4)


def nccl_unique_id() -> bytes:
    """sage_nccl_unique_id: 128 bytes to broadcast from rank 0 to every rank."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().sage_nccl_unique_id(buf))
    return buf.raw


def debug_loopback_id(world: int) -> bytes:
    """sage_debug_loopback_id (tests only): an id for ``world`` logical ranks on this one GPU."""
    buf = ctypes.create_string_buffer(128)
    _check(lib().sage_debug_loopback_id(int(world), buf))
    return buf.raw


def load_csr(off, col, w=None, n: int | None = None, symmetric: bool = False, push_only: bool = False,
             borrow: bool = False, validate: bool = True, tile_cta: int = 256, tile_min: int = 8,
             align: int = 4, alpha: float = 15.0, beta: float = 18.0, stream=None, ctas_per_sm: int = 0,
             hub_filter: int = 0,
             rank: int = 0, world: int = 1, nccl_unique_id: bytes | None = None,
             v_begin: int = 0, v_end: int | None = None, host_columns: bool = False,
             exchange: int = 0) -> Graph:
    """sage_load_csr.  ``off``/``col``/``w`` are host arrays or tensors, or CUDA tensors."""
    po, ko, dev_o = _ptr(off, np.int64)
    pc, kc, dev_c = _ptr(col, np.int32)
    pw, kw, dev_w = _ptr(w, np.uint32)
    devs = {dev_o, dev_c} | ({dev_w} if w is not None else set())
    if len(devs) != 1:
        raise TypeError("row_offsets, col_indices and weights must all be host or all be device arrays")
    dev = dev_o
    n_rows = len(off) - 1
    flags = (F_SYMMETRIC if symmetric else 0) | (F_PUSH_ONLY if push_only else 0)
    if dev:
        flags |= F_DEVICE_PTRS | (F_BORROW if borrow else 0)
    if not validate:
        flags |= F_NO_VALIDATE
    if host_columns:
        flags |= F_HOST_COLUMNS | (F_BORROW if borrow else 0)
    csr = Csr()
    csr.n = int(n if n is not None else n_rows)
    csr.m = int(len(col))
    csr.row_offsets = po
    csr.col_indices = pc
    csr.weights = pw
    csr.flags = flags
    if stream is None and dev:
        # device inputs: order the library's work after the caller's producing work (torch stream)
        import torch
        stream = torch.cuda.current_stream().cuda_stream
    csr.cuda_stream = stream
    opts = Options(tile_cta, tile_min, align, alpha, beta, ctas_per_sm, hub_filter)
    csr.opts = ctypes.pointer(opts)
    dist = None
    if nccl_unique_id is not None:
        idbuf = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
        dist = Dist(rank, world, ctypes.cast(idbuf, ctypes.c_void_p).value, v_begin,
                    v_end if v_end is not None else csr.n, exchange)
        csr.dist = ctypes.pointer(dist)
    h = ctypes.c_void_p()
    _check(lib().sage_load_csr(ctypes.byref(csr), ctypes.byref(h)))
    return Graph(h.value, (ko, kc, kw) if borrow else None)
