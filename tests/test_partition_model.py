"""CPU model of the multi-GPU protocol, run with world_size 2 on gloo.

TEST MODEL, not a backend: pure numpy, one process per logical rank, torch.distributed (gloo,
127.0.0.1) standing in for NCCL.  It mirrors the host-side logic of csrc/comm.cu step by step —
1D contiguous blocks, the padded global index r*P + (v - vb[r]), push levels with a dense
candidate bitmap exchanged to the owners, owners applying candidates, the (|F|, arcs(F))
allreduce driving termination and the Beamer direction, the frontier allgather before pull
levels, PageRank's reduce-scatter of partial sums plus the dangling allreduce, and SSSP's
min reduce-scatter of remote candidate distances per Bellman-Ford iteration — and checks the
gathered answers against the oracle.
"""
import os
import socket

import numpy as np
import pytest

import oracle
import sagegen as sg


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _blocks(n, world):
    b = [n * r // world for r in range(world + 1)]
    return b


class Part:
    def __init__(self, rank, world, n):
        self.rank, self.world = rank, world
        self.vb = _blocks(n, world)
        maxrows = max(self.vb[r + 1] - self.vb[r] for r in range(world))
        self.P = 32 * ((maxrows + 31) // 32 + 1)

    def owner(self, v):
        return int(np.searchsorted(self.vb, v, side="right") - 1)

    def pidx(self, v):
        r = self.owner(v)
        return r * self.P + (v - self.vb[r]), r == self.rank


def _allreduce(x, dist):
    import torch
    t = torch.tensor(x, dtype=torch.float64)
    dist.all_reduce(t)
    return t.numpy()


def _allgather(arr, dist, world):
    import torch
    t = torch.from_numpy(np.ascontiguousarray(arr))
    out = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(out, t)
    return [o.numpy() for o in out]


def model_bfs(rank, world, g, src, dist, alpha=15.0, beta=18.0, direction=True):
    pm = Part(rank, world, g.n)
    vb, ve = pm.vb[rank], pm.vb[rank + 1]
    nl = ve - vb
    deg = np.diff(g.off)
    visited = np.zeros(world * pm.P, dtype=bool)       # own slice authoritative, remote = "sent"
    level = np.full(nl, -1, dtype=np.int32)
    frontier = []
    fb = np.zeros(world * pm.P, dtype=bool)
    if vb <= src < ve:
        level[src - vb] = 0
        visited[pm.pidx(src)[0]] = True
        fb[pm.pidx(src)[0]] = True
        frontier = [src - vb]
    seed_arcs = _allreduce([sum(deg[vb + u] for u in frontier)], dist)[0]
    m_total = _allreduce([float(g.off[ve] - g.off[vb])], dist)[0]
    mU = m_total - seed_arcs
    dir_, prev = 0, 1
    L = 0
    while True:
        nxt, fbn = [], np.zeros(world * pm.P, dtype=bool)
        if dir_ == 0:
            out = np.zeros(world * pm.P, dtype=bool)
            for u in frontier:
                for v in g.col[g.off[vb + u]:g.off[vb + u + 1]]:
                    p, own = pm.pidx(int(v))
                    if visited[p]:
                        continue
                    visited[p] = True
                    if own:
                        level[v - vb] = L + 1
                        nxt.append(v - vb)
                        fbn[p] = True
                    else:
                        out[p] = True
            # dense "alltoall": each owner takes its slice of every rank's candidate bitmap
            allout = _allgather(out.astype(np.uint8), dist, world)
            lo = rank * pm.P
            cand = np.zeros(pm.P, dtype=bool)
            for r in range(world):
                if r != rank:
                    cand |= allout[r][lo:lo + pm.P].astype(bool)
            cand[nl:] = False
            new = np.nonzero(cand & ~visited[lo:lo + pm.P])[0]
            for lv in new:
                visited[lo + lv] = True
                fbn[lo + lv] = True
                level[lv] = L + 1
                nxt.append(int(lv))
        else:
            lo = rank * pm.P
            for v in range(nl):
                if visited[lo + v]:
                    continue
                for u in g.col[g.off[vb + v]:g.off[vb + v + 1]]:
                    if fb[pm.pidx(int(u))[0]]:
                        visited[lo + v] = True
                        fbn[lo + v] = True
                        level[v] = L + 1
                        nxt.append(v)
                        break
        nF, aF = _allreduce([float(len(nxt)), float(sum(deg[vb + u] for u in nxt))], dist)
        if nF == 0:
            break
        mU -= aF
        ndir = dir_
        if direction:
            if dir_ == 0 and aF > mU / alpha:
                ndir = 1
            elif dir_ == 1 and not (nF >= prev or nF > g.n / beta):
                ndir = 0
        if ndir == 1:      # allgather of every owner's frontier slice
            parts = _allgather(fbn.astype(np.uint8), dist, world)
            fbn = np.zeros(world * pm.P, dtype=bool)
            for r in range(world):
                fbn[r * pm.P:(r + 1) * pm.P] = parts[r][r * pm.P:(r + 1) * pm.P].astype(bool)
        fb, frontier, dir_, prev = fbn, nxt, ndir, nF
        L += 1
    return level


def model_pagerank(rank, world, g, dist, d=0.85, iters=20):
    pm = Part(rank, world, g.n)
    vb, ve = pm.vb[rank], pm.vb[rank + 1]
    nl = ve - vb
    x = np.full(nl, 1.0 / g.n)
    for _ in range(iters):
        y = np.zeros(world * pm.P)
        D = 0.0
        for u in range(nl):
            b, e = g.off[vb + u], g.off[vb + u + 1]
            if e == b:
                D += x[u]
                continue
            for v in g.col[b:e]:
                y[pm.pidx(int(v))[0]] += x[u] / (e - b)
        ysum = _allreduce(y, dist)                       # reduce-scatter = allreduce + own slice
        yown = ysum[rank * pm.P:rank * pm.P + nl]
        Dg = _allreduce([D], dist)[0]
        x = (1 - d) / g.n + d * (yown + Dg / g.n)
    return x


def model_sssp(rank, world, g, w, src, dist):
    """csrc/comm.cu run_sssp_multi: own targets relaxed in place, remote ones min-ed into the padded
    candidate array, ncclReduceScatter(min) to the owners, owners apply, |improved| allreduce."""
    import torch
    pm = Part(rank, world, g.n)
    vb, ve = pm.vb[rank], pm.vb[rank + 1]
    nl = ve - vb
    INF = 0xFFFFFFFF
    d = np.full(nl, INF, dtype=np.uint64)
    frontier = []
    if vb <= src < ve:
        d[src - vb] = 0
        frontier = [src - vb]
    while True:
        cand = np.full(world * pm.P, INF, dtype=np.int64)
        inq = set()
        for u in frontier:
            du = int(d[u])
            for k in range(g.off[vb + u], g.off[vb + u + 1]):
                nd = du + int(w[k])
                assert nd < INF
                p, own = pm.pidx(int(g.col[k]))
                if own:
                    lv = int(g.col[k]) - vb
                    if nd < d[lv]:
                        d[lv] = nd
                        inq.add(lv)
                elif nd < cand[p]:
                    cand[p] = nd
        t = torch.from_numpy(cand)
        dist.all_reduce(t, op=dist.ReduceOp.MIN)          # reduce-scatter(min) = allreduce + own slice
        cown = t.numpy()[rank * pm.P:rank * pm.P + nl]
        for lv in np.nonzero(cown < d.astype(np.int64))[0]:
            d[lv] = cown[lv]
            inq.add(int(lv))
        nF = _allreduce([float(len(inq))], dist)[0]
        if nF == 0:
            break
        frontier = sorted(inq)
    return d.astype(np.uint32)


def _worker(rank, world, port, outdir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res = {}
    for k, (scale, sym) in enumerate([(9, True), (9, False), (10, True)]):
        g = sg.rmat(scale, 8, seed=k + 1, symmetric=sym)
        for s in sg.sources(g, 2, seed=2):
            res[f"bfs{k}_{int(s)}_do"] = model_bfs(rank, world, g, int(s), dist, direction=sym)
            res[f"bfs{k}_{int(s)}_push"] = model_bfs(rank, world, g, int(s), dist, direction=False)
    g = sg.rmat(8, 8, seed=7, symmetric=False)
    res["pr"] = model_pagerank(rank, world, g, dist)
    for k, sym in enumerate([True, False]):
        g = sg.rmat(9, 8, seed=11 + k, symmetric=sym)
        w = sg.weights(g, 1)
        for s in sg.sources(g, 2, seed=2):
            res[f"sssp{k}_{int(s)}"] = model_sssp(rank, world, g, w, int(s), dist)
    np.savez(os.path.join(outdir, f"rank{rank}.npz"), **res)
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partitioned_protocol_matches_oracle(tmp_path, world):
    import torch.multiprocessing as mp
    port = _free_port()
    mp.spawn(_worker, args=(world, port, str(tmp_path)), nprocs=world, join=True)
    parts = [np.load(os.path.join(tmp_path, f"rank{r}.npz")) for r in range(world)]
    for k, (scale, sym) in enumerate([(9, True), (9, False), (10, True)]):
        g = sg.rmat(scale, 8, seed=k + 1, symmetric=sym)
        for s in sg.sources(g, 2, seed=2):
            ref = oracle.bfs(g.off, g.col, int(s))
            for mode in ("do", "push"):
                got = np.concatenate([p[f"bfs{k}_{int(s)}_{mode}"] for p in parts])
                assert np.array_equal(got, ref), (k, int(s), mode)
    g = sg.rmat(8, 8, seed=7, symmetric=False)
    x = np.concatenate([p["pr"] for p in parts])
    xr = oracle.pagerank(g.off, g.col, 0.85, 20)
    assert np.max(np.abs(x - xr) / xr) < 1e-12
    for k, sym in enumerate([True, False]):
        g = sg.rmat(9, 8, seed=11 + k, symmetric=sym)
        w = sg.weights(g, 1)
        for s in sg.sources(g, 2, seed=2):
            ref, _ = oracle.sssp(g.off, g.col, w, int(s))
            got = np.concatenate([p[f"sssp{k}_{int(s)}"] for p in parts])
            assert np.array_equal(got, ref), (k, int(s))
