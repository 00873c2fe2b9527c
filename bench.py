#!/usr/bin/env python
"""SAGE hot-path benchmark (BASELINE.json metric: BFS/SSSP GTEPS, fraction of HBM roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C2]

One step = one BFS query (the paper's push expansion: Tiled Partitioning + Resident Tile
Stealing, SAGE_F_PUSH_ONLY) from the next seeded source on the workload BASELINE.json quotes its
metric on that fits one GPU: configs[1] = RMAT scale-24 (Graph500 Kronecker, edgefactor 16,
symmetrised, weighted).  W untimed warm-up steps, then K timed steps, each bracketed by CUDA
events on the graph's stream; L2 is flushed (256 MB write) between steps.  Rank 0 prints ONE JSON
line.  Extra keys carry SSSP, direction-optimising BFS and PageRank on the same graph, the
roofline of the dominant kernel (the persistent traversal kernel), the timed CPU oracle and an
end-to-end number through the C ABI with host buffers.

--impl reference runs the CPU oracle (oracle/, serial C) on the same config and metric.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "BFS GTEPS (push TP+RTS, RMAT-24)"


def _args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=8)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="C2")
    p.add_argument("--scale", type=int, default=None, help="override the RMAT scale (debug only)")
    p.add_argument("--no-extras", action="store_true")
    p.add_argument("--nccl", action="store_true", help="use the multi-GPU (NCCL) path even at N=1")
    return p.parse_args()


def _graph(cfg, scale):
    import sagegen as sg
    if scale is not None:
        g = sg.rmat(scale, 16, 1, True)
        g.w = sg.weights(g, 1)
        return g, f"rmat{scale}_sym_ef16_seed1"
    g = sg.config(cfg)
    return g, {"C1": "rmat16_sym_ef16_seed1", "C2": "rmat24_sym_ef16_seed1_w255"}.get(cfg, cfg)


class Clocks:
    """nvidia-smi sampler running during the timed region."""

    def __init__(self, gpu: int):
        self.samples = []
        self.proc = None
        self.gpu = gpu

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        time.sleep(0.25)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        time.sleep(0.2)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if len(s) > i + 2 and s[i + 2].lower().startswith("active")})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback"


def _traffic():
    """dram bytes per launch of the persistent BFS kernel from the committed ncu --set full capture."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        return d
    except Exception:
        return None


def _pin_one_core():
    """SURVEY §8(d) oracle timing: the serial oracle runs pinned to one host core; returns a
    description of the host (CPU model, cores) for the cpu_baseline object."""
    try:
        cpus = sorted(os.sched_getaffinity(0))
        os.sched_setaffinity(0, {cpus[-1]})
    except Exception:
        pass
    model = "unknown CPU"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return model, os.cpu_count()


def _unpin():
    try:
        os.sched_setaffinity(0, set(range(os.cpu_count())))
    except Exception:
        pass


def _dist():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def run_reference(a):
    """The CPU oracle (serial C) on the same workload: each step = one oracle BFS."""
    rank, world, _ = _dist()
    if rank != 0:
        return
    import oracle
    import sagegen as sg
    g, gname = _graph(a.config, a.scale)
    srcs = sg.sources(g, a.warmup + a.steps, seed=2)
    deg = np.diff(g.off)
    model, ncpu = _pin_one_core()
    times, edges = [], []
    for i, s in enumerate(srcs):
        t0 = time.perf_counter()
        lv = oracle.bfs(g.off, g.col, int(s))
        dt = time.perf_counter() - t0
        if i >= a.warmup:
            times.append(dt)
            edges.append(int(deg[lv >= 0].sum()) // 2)
    gteps = [e / t / 1e9 for e, t in zip(edges, times)]
    hm = len(gteps) / sum(1 / x for x in gteps)
    line = {"metric": METRIC, "value": hm, "unit": "GTEPS", "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": 1e3 * float(np.mean(times)), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": gname, "n": g.n, "arcs": g.m, "mode": "serial FIFO BFS (oracle/oracle.c)"},
            "cpu_baseline": {"value": hm, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                             "sample": f"{a.steps} timed oracle BFS sources of {gname} after {a.warmup} warm-up",
                             "host": f"serial oracle, 1 core of {model}, host has {ncpu} cores"},
            "e2e": {"value": hm, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def _spawn_if_needed(a):
    """`python bench.py --gpus N` with N > 1 outside torchrun: re-launch as N ranks (one process
    per GPU) through torch.distributed.run on 127.0.0.1; returns the child's exit code, or None
    when this process is already a rank (or N == 1)."""
    if a.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return None
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def multi_workload(config: str, world: int):
    """Kronecker scale of the multi-GPU runs (weak scaling: per-GPU work fixed as N grows).
    Default: 24 + log2(N) (N = 1 is C2's scale); --config C5: 27 + log2(N) (Kron-30 at N = 8,
    SURVEY §8(d) C5).  N must be a power of two."""
    lg = world.bit_length() - 1
    if 1 << lg != world:
        raise ValueError("the multi-GPU bench needs a power-of-two number of ranks")
    base = 27 if config == "C5" else 24
    return base + lg


def _nonempty_sources(torch, off_d, n, world, k, seed=2):
    """sagegen.sources' rule (uniform over vertices with out-degree > 0, seeded hash tries) on a
    1D-partitioned graph: the per-rank 'row non-empty' flags are allgathered."""
    import sagegen as sg
    ne = (off_d[1:] > off_d[:-1]).to(torch.uint8)
    if world > 1:
        parts = [torch.empty_like(ne) for _ in range(world)]
        torch.distributed.all_gather(parts, ne)
        ne = torch.cat(parts)
    out = []
    for i in range(k):
        for j0 in range(0, 1 << 20, 64):
            cand = torch.tensor([sg.hash3(seed, i, j) % n for j in range(j0, j0 + 64)], dtype=torch.int64,
                                device=ne.device)
            hit = torch.nonzero(ne[cand]).flatten()
            if len(hit):
                out.append(int(cand[int(hit[0])]))
                break
    return np.array(out, dtype=np.int32)


def main():
    a = _args()
    if a.impl == "reference":
        run_reference(a)
        return
    rc = _spawn_if_needed(a)
    if rc is not None:
        sys.exit(rc)
    import torch

    import paper_conf_sigmod_00020t21_b200 as sage
    import sagegen as sg
    from __graft_entry__ import build

    rank, world, local = _dist()
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    build()
    stream = torch.cuda.Stream()   # one dedicated stream: the library's work, the L2 flush and the
    torch.cuda.set_stream(stream)  # timing events are all ordered on it
    multi = world > 1 or a.nccl
    if not multi:
        g, gname = _graph(a.config, a.scale)
        off_d = torch.from_numpy(g.off).cuda()
        col_d = torch.from_numpy(g.col).cuda()
        w_d = torch.from_numpy(g.w).cuda() if g.w is not None else None
        G = sage.load_csr(off_d, col_d, w_d, symmetric=True, borrow=True, stream=stream.cuda_stream)
        n = g.n
        n_rows = n
    else:
        # every rank generates its own 1D block of the Kronecker graph on its GPU (all tuples
        # regenerated, arcs of other owners dropped: sagegen/sagegen_dev.cu), no host graph
        scale = a.scale if a.scale is not None else multi_workload(a.config, world)
        n = 1 << scale
        vb, ve = n * rank // world, n * (rank + 1) // world
        off_d, col_d, w_d = sg.rmat_device(scale, 16, 1, True, vb, ve, weights_seed=1)
        if world > 1:
            obj = [sage.nccl_unique_id() if rank == 0 else None]
            torch.distributed.broadcast_object_list(obj, 0)
            uid = obj[0]
        else:
            uid = sage.nccl_unique_id()
        m_all = torch.tensor([col_d.numel()], dtype=torch.int64, device="cuda")
        if world > 1:
            torch.distributed.all_reduce(m_all)
        gname = f"kron{scale}_sym_ef16_seed1_w255" + ("_C5" if a.config == "C5" else "")
        G = sage.load_csr(off_d, col_d, w_d, n=n, symmetric=True, borrow=True, stream=stream.cuda_stream,
                          rank=rank, world=world, nccl_unique_id=uid, v_begin=vb, v_end=ve)
        n_rows = ve - vb

        class _G:   # what the rest of main needs of the workload
            pass
        g = _G()
        g.n, g.m, g.w = n, int(m_all.item()), None
        g.srcs = _nonempty_sources(torch, off_d, n, world, a.warmup + a.steps)
    srcs = g.srcs if multi else sg.sources(g, a.warmup + a.steps, seed=2)
    level = torch.empty(n_rows, dtype=torch.int32, device="cuda")
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
            torch.cuda.synchronize()

    # ---------------- headline: push-only BFS (TP + RTS), K timed steps
    for i in range(a.warmup):
        G.bfs(int(srcs[i]), out=level, push_only=True)
    stats = []
    times = []
    with Clocks(local) as ck:
        barrier()
        for i in range(a.warmup, a.warmup + a.steps):
            flush.fill_(float(i))
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            _, _, st = G.bfs(int(srcs[i]), out=level, push_only=True)
            e1.record(stream)
            e1.synchronize()
            times.append(e0.elapsed_time(e1))
            stats.append(st)
        barrier()
    clocks = ck.summary()
    t_max = float(np.sum(times))
    if world > 1:
        tt = torch.tensor([t_max], device="cuda")
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        t_max = float(tt.item())
    edges = [s["edges_traversed"] for s in stats]
    gteps = [e / (t * 1e-3) / 1e9 for e, t in zip(edges, times)]
    hm = len(gteps) / sum(1 / x for x in gteps)
    if world > 1:   # global edges over the max-over-ranks time of each step
        tt = torch.tensor(times, device="cuda")
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        times = tt.cpu().tolist()
        gteps = [e / (t * 1e-3) / 1e9 for e, t in zip(edges, times)]
        hm = len(gteps) / sum(1 / x for x in gteps)
    value = hm
    kms = float(np.mean([s["kernel_ms"] for s in stats]))
    kbytes = float(np.mean([s["model_bytes"] - 4.0 * n for s in stats]))
    peaks, peak_src = _peaks()
    achieved = kbytes / (kms * 1e-3) / 1e9
    tr = _traffic()
    st_last = stats[-1]
    # SURVEY §8(d) compulsory floor: 4 B per inspected arc + 16 B per expanded vertex + 4n B
    floor = 4.0 * st_last["arcs_inspected"] + 16.0 * st_last["vertices_expanded"] + 4.0 * n
    traffic = (tr or {}).get("bfs_push_bytes_per_launch")
    roof = {"bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
            "frac": achieved / peaks["hbm_gbs"], "traffic": traffic,
            "traffic_source": (tr or {}).get("source", "none") + " — an ncu --set full capture of this kernel on "
                              "this workload, committed under profiles/; not measured inside this run",
            "frac_nominal_8TBps": achieved / 8000.0,
            "amplification": (traffic / kbytes) if traffic else None,
            "l2_hit_rate_pct": (tr or {}).get("lts_hit_rate_pct"),
            "compulsory_floor_bytes": floor,
            "floor_frac": floor / (kms * 1e-3) / 1e9 / peaks["hbm_gbs"],
            "kernel": ("k_bfs_fused_hub<4,3> (persistent fused runtime-TP + RTS consumer)" if not multi else
                       "host-sequenced levels (k_mpush + " + ("peer-memory inbox ORs + barrier" if G.peer_exchange
                                                              else "NCCL all-to-all(v)")
                       + " + k_mapply), time incl. exchange"),
            "peak_source": peak_src,
            "model": "SURVEY §8(d): 20 B/expanded vertex + 8 B/inspected arc + 8 B/discovered vertex",
            "kernel_ms": kms, "model_bytes_per_launch": kbytes}
    line = {"metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": t_max / a.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": gname, "n": n, "arcs": g.m, "mode": "push-only (SAGE_F_PUSH_ONLY)",
                       "tile_ladder": "B=256 M=8 A=4", "l2": "flushed between steps (256 MB write)",
                       "parallelism": f"1D-partition x{world} (NCCL)" if multi else "single",
                       **({"generated": ("per rank on device (sagegen_dev); weak scaling, Kronecker scale "
                                         + ("27" if a.config == "C5" else "24") + " + log2(N)")}
                          if multi else {})},
            "gpu_launches": (2 * a.steps if not multi else
                             sum(2 + s["levels"] * (3 if world > 1 else 2) for s in stats)),
            "clocks": clocks, "roofline": roof,
            "bfs_levels": stats[-1]["levels"]}
    if rank == 0 and not a.no_extras and not multi:
        line.update(_extras(a, G, g, srcs, level, flush, stream, sage))
    if multi:
        line["sssp"] = _sssp_multi(a, G, srcs, n_rows, world, flush, stream)
        line["e2e"] = _e2e_multi(a, G, g, srcs, sage, rank, world, off_d, col_d, n, uid if world == 1 else None)
    if rank == 0:
        print(json.dumps(line), flush=True)
    G.free()
    if world > 1:
        torch.distributed.destroy_process_group()


def _sssp_multi(a, G, srcs, n_rows, world, flush, stream):
    """Multi-GPU SSSP (min reduce-scatter per Bellman-Ford iteration): GTEPS over up to 4 sources,
    each step's time = max over ranks."""
    import torch
    dist = torch.empty(n_rows, dtype=torch.uint32, device="cuda")
    G.sssp(int(srcs[0]), out=dist)
    times, edges, iters = [], [], []
    for i in range(min(4, a.steps)):
        flush.fill_(float(i))
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        _, st = G.sssp(int(srcs[a.warmup + i]), out=dist)
        times.append(st["ms"])
        edges.append(st["edges_traversed"])
        iters.append(st["levels"])
    if world > 1:
        tt = torch.tensor(times, device="cuda")
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        times = tt.cpu().tolist()
    g = [e / (t * 1e-3) / 1e9 for e, t in zip(edges, times)]
    return {"gteps": len(g) / sum(1 / x for x in g), "ms": float(np.median(times)),
            "iterations": int(np.median(iters)), "sources": len(g),
            "exchange": "ncclReduceScatter(min) of candidate distances per iteration"}


def _e2e_multi(a, G, g, srcs, sage, rank, world, off_d, col_d, n, uid):
    """End to end on the NCCL path: every rank loads its block from pinned host memory (H2D),
    runs the BFS, reads its level slice back (D2H); time = max over ranks."""
    import torch
    off_h = off_d.cpu().pin_memory()
    col_h = col_d.cpu().pin_memory()
    lv_h = torch.empty(len(off_h) - 1, dtype=torch.int32).pin_memory()
    vb, ve = G.v_begin, G.v_begin + G.n_local
    res = []
    for i in range(2):
        if world > 1:
            obj = [sage.nccl_unique_id() if rank == 0 else None]
            torch.distributed.broadcast_object_list(obj, 0)
            u = obj[0]
            torch.distributed.barrier()
        else:
            u = sage.nccl_unique_id()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with sage.load_csr(off_h, col_h, n=n, symmetric=True, rank=rank, world=world, nccl_unique_id=u,
                           v_begin=vb, v_end=ve) as H:
            _, _, st = H.bfs(int(srcs[i]), out=lv_h, push_only=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        if world > 1:
            t = torch.tensor([dt], device="cuda")
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            dt = float(t.item())
        res.append((dt, st["edges_traversed"]))
    return {"value": len(res) / sum(t * 1e9 / e for t, e in res), "unit": "GTEPS",
            "h2d_bytes_per_step": int(off_h.numel() * 8 + col_h.numel() * 4),
            "d2h_bytes_per_step": int(lv_h.numel() * 4),
            "includes": "per rank: sage_load_csr of its block from pinned host memory (copy + validation + "
                        "NCCL communicator) + sage_bfs + level D2H; max over ranks"}


def _time_calls(fn, k, flush, stream):
    import torch
    out = []
    for i in range(k):
        flush.fill_(float(i))
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        st = fn(i)
        e1.record(stream)
        e1.synchronize()
        out.append((e0.elapsed_time(e1), st))
    return out


def _lv_in_core(G, src, level_ooc):
    """Levels of the out-of-core run (already in ``level_ooc``) vs the in-core graph."""
    import torch
    ooc = level_ooc.cpu().numpy().copy()
    ref = torch.empty_like(level_ooc)
    G.bfs(int(src), out=ref, push_only=True)
    return np.array_equal(ooc, ref.cpu().numpy())


def _extras(a, G, g, srcs, level, flush, stream, sage):
    import torch

    import oracle
    ex = {}
    k = max(2, min(a.steps, 4))
    # direction-optimising BFS
    G.bfs(int(srcs[0]), out=level)
    r = _time_calls(lambda i: G.bfs(int(srcs[i]), out=level)[2], k, flush, stream)
    ex["bfs_do"] = {"gteps": len(r) / sum(t * 1e-3 * 1e9 / st["edges_traversed"] for t, st in r),
                    "ms": float(np.mean([t for t, _ in r])), "pull_levels": r[-1][1]["pull_levels"],
                    "arcs_inspected_frac": r[-1][1]["arcs_inspected"] / g.m}
    # SSSP
    dist = torch.empty(g.n, dtype=torch.int32, device="cuda").view(torch.uint32)
    G.sssp(int(srcs[0]), out=dist)                 # warm-up (first call allocates SSSP state)
    r = _time_calls(lambda i: G.sssp(int(srcs[i]), out=dist)[1], k, flush, stream)
    ex["sssp"] = {"gteps": len(r) / sum(t * 1e-3 * 1e9 / st["edges_traversed"] for t, st in r),
                  "ms": float(np.mean([t for t, _ in r])), "iterations": r[-1][1]["levels"],
                  "arcs_relaxed_per_edge": r[-1][1]["arcs_inspected"] / g.m,
                  "model_GBps": float(np.mean([st["model_bytes"] / (st["kernel_ms"] * 1e-3) / 1e9 for _, st in r]))}
    # Betweenness Centrality (NEXT #1): one source = forward sigma BFS + backward delta sweep
    bcv = torch.empty(g.n, dtype=torch.float64, device="cuda")
    G.bc([int(srcs[0])], out=bcv)
    r = _time_calls(lambda i: G.bc([int(srcs[i])], out=bcv)[1], k, flush, stream)
    ex["bc"] = {"ms_per_source": float(np.mean([t for t, _ in r])),
                "gteps": len(r) / sum(t * 1e-3 * 1e9 / st["edges_traversed"] for t, st in r),
                "note": "edges = reached undirected edges of the source; both passes inside the time"}
    # PageRank 20 iterations: pull (default on symmetric graphs) and the paper's push form
    x = torch.empty(g.n, dtype=torch.float64, device="cuda")
    ex["pagerank"] = {}
    for form, po in (("pull", False), ("push", True)):
        G.pagerank(0.85, 20, out=x, push_only=po)
        r = _time_calls(lambda i: G.pagerank(0.85, 20, out=x, push_only=po)[1], 2, flush, stream)
        ms = float(np.mean([t for t, _ in r]))
        ex["pagerank"][form] = {"ms_20_iter": ms, "gedges_per_s": 20 * g.m / (ms * 1e-3) / 1e9,
                                "model_GBps": float(np.mean([st["model_bytes"] / (st["kernel_ms"] * 1e-3) / 1e9
                                                             for _, st in r]))}
    # C4 shape (UK-like: directed, crawl order, tendrils -> ~500 levels) at 10M vertices:
    # push-only BFS (tail mode on the long small-frontier stretch) and PageRank (push)
    import sagegen as sg
    uk = sg.uk_like(n=10_000_000, seed=1, n_tendrils=200)
    with sage.load_csr(torch.from_numpy(uk.off).cuda(), torch.from_numpy(uk.col).cuda(),
                       stream=stream.cuda_stream) as U:
        lvu = torch.empty(uk.n, dtype=torch.int32, device="cuda")
        us = sg.sources(uk, 3, seed=2)
        U.bfs(int(us[0]), out=lvu)
        r = _time_calls(lambda i: U.bfs(int(us[1 + i % 2]), out=lvu)[2], 2, flush, stream)
        xu = torch.empty(uk.n, dtype=torch.float64, device="cuda")
        U.pagerank(0.85, 20, out=xu)
        rp = _time_calls(lambda i: U.pagerank(0.85, 20, out=xu)[1], 1, flush, stream)
        ex["c4_shape"] = {"graph": f"uk_like n={uk.n} arcs={uk.m} (C4 shape at 1/10.5 size)",
                          "bfs_ms": float(np.mean([t for t, _ in r])), "bfs_levels": r[-1][1]["levels"],
                          "bfs_gteps": len(r) / sum(t * 1e-3 * 1e9 / st["edges_traversed"] for t, st in r),
                          "pagerank_ms_20_iter": rp[0][0],
                          "pagerank_form": "windowed push" if U.pagerank_windowed else "log-based push"}
        U.pagerank(0.85, 20, out=xu, stealing=False)
        rl = _time_calls(lambda i: U.pagerank(0.85, 20, out=xu, stealing=False)[1], 1, flush, stream)
        ex["c4_shape"]["pagerank_log_form_ms_20_iter"] = rl[0][0]
    # out-of-core (NEXT #4): C2 with col in pinned host memory read zero-copy over the host link
    # (copied into library-owned pinned memory at load); push and DO BFS, parity checked
    with sage.load_csr(g.off, g.col, symmetric=True, host_columns=True, align=32,
                       stream=stream.cuda_stream) as O:
        oo = {}
        for form, po in (("push", True), ("do", False)):
            O.bfs(int(srcs[0]), out=level, push_only=po)
            r = _time_calls(lambda i: O.bfs(int(srcs[i]), out=level, push_only=po)[2], 2, flush, stream)
            oo[form] = {"ms": float(np.mean([t for t, _ in r])),
                        "gteps": len(r) / sum(t * 1e-3 * 1e9 / st["edges_traversed"] for t, st in r)}
        O.bfs(int(srcs[0]), out=level, push_only=True)
        oo["levels_equal_in_core"] = bool(_lv_in_core(G, srcs[0], level))
        oo["note"] = "col (2.08 GB) in pinned host memory; tile alignment 32 (128-B requests)"
        ex["out_of_core"] = oo
    # C1 (BASELINE configs[0]): RMAT-16, L2-resident and launch/latency-bound; 16 sources, push
    # and direction-optimising, each checked against the oracle, which is timed beside it
    c1 = sg.config("C1")
    with sage.load_csr(torch.from_numpy(c1.off).cuda(), torch.from_numpy(c1.col).cuda(), symmetric=True,
                       stream=stream.cuda_stream) as C:
        lv1 = torch.empty(c1.n, dtype=torch.int32, device="cuda")
        s1 = sg.sources(c1, 16, seed=2)
        res = {}
        for form, po in (("push", True), ("do", False)):
            C.bfs(int(s1[0]), out=lv1, push_only=po)
            r = _time_calls(lambda i: C.bfs(int(s1[i]), out=lv1, push_only=po)[2], len(s1), flush, stream)
            ok = True
            for i in range(4):
                C.bfs(int(s1[i]), out=lv1, push_only=po)
                ok &= bool(np.array_equal(lv1.cpu().numpy(), oracle.bfs(c1.off, c1.col, int(s1[i]))))
            res[form] = {"us_median": float(np.median([t for t, _ in r])) * 1e3,
                         "gteps": len(r) / sum(t * 1e-3 * 1e9 / st["edges_traversed"] for t, st in r),
                         "levels_equal_oracle_4_sources": ok}
        t0 = time.perf_counter()
        for i in range(16):
            oracle.bfs(c1.off, c1.col, int(s1[i]))
        to = (time.perf_counter() - t0) / 16
        res["oracle_us_per_source"] = to * 1e6
        res["roofline"] = "n/a (graph L2-resident: latency / launch bound, SURVEY 8(d))"
        ex["c1"] = res
    # end-to-end through the C ABI with HOST buffers: load (H2D) + BFS + level D2H
    off_h = torch.from_numpy(g.off).pin_memory()
    col_h = torch.from_numpy(g.col).pin_memory()
    lv_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
    e2e = []
    for i in range(3):   # step 0 = untimed warm-up (memory-pool growth after the extras above)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with sage.load_csr(off_h, col_h, symmetric=True) as H:
            _, _, st = H.bfs(int(srcs[i]), out=lv_h, push_only=True)
        torch.cuda.synchronize()
        if i:
            e2e.append((time.perf_counter() - t0, st["edges_traversed"]))
    ex["e2e"] = {"value": len(e2e) / sum(t * 1e9 / e for t, e in e2e), "unit": "GTEPS",
                 "ms_per_step": float(np.mean([t for t, _ in e2e])) * 1e3, "warmup": 1, "steps": len(e2e),
                 "h2d_bytes_per_step": int(g.off.nbytes + g.col.nbytes), "d2h_bytes_per_step": int(4 * g.n),
                 "includes": "sage_load_csr from pinned host CSR (copy + validation) + sage_bfs + level D2H"}
    # timed CPU oracle on a bounded sample of the same workload (serial, pinned to one
    # core, 8 BFS and 4 SSSP sources at C2), also the full-size parity check of those sources
    import sagegen as sg
    osrc = sg.sources(g, 8, seed=2)    # the first 8 bench sources (same seeded rule)
    gpu_lv, gpu_d = [], []
    for i in range(8):
        G.bfs(int(osrc[i]), out=level, push_only=True)
        gpu_lv.append(level.cpu().numpy().copy())
    for i in range(4):
        G.sssp(int(osrc[i]), out=dist)
        gpu_d.append(dist.cpu().numpy().view(np.uint32).copy())
    model, ncpu = _pin_one_core()
    deg = np.diff(g.off)
    bt, be, st_, se = [], [], [], []
    bfs_ok = sssp_ok = True
    for i in range(8):
        t0 = time.perf_counter()
        lv = oracle.bfs(g.off, g.col, int(osrc[i]))
        bt.append(time.perf_counter() - t0)
        be.append(int(deg[lv >= 0].sum()) // 2)
        bfs_ok &= bool(np.array_equal(lv, gpu_lv[i]))
    for i in range(4):
        t0 = time.perf_counter()
        dd, _ = oracle.sssp(g.off, g.col, g.w, int(osrc[i]))
        st_.append(time.perf_counter() - t0)
        se.append(int(deg[dd != 0xFFFFFFFF].sum()) // 2)
        sssp_ok &= bool(np.array_equal(dd, gpu_d[i]))
    _unpin()
    hb = len(bt) / sum(t * 1e9 / e for t, e in zip(bt, be))
    hs = len(st_) / sum(t * 1e9 / e for t, e in zip(st_, se))
    ex["cpu_baseline"] = {"value": hb, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                          "sample": "8 serial oracle BFS (oracle/oracle.c FIFO queue) of the bench sources, "
                                    "harmonic mean; 4 Dijkstra SSSP beside it",
                          "seconds": sum(bt), "sssp_gteps": hs, "sssp_seconds": sum(st_),
                          "host": f"serial oracle, 1 core of {model}, host has {ncpu} cores"}
    ex["parity"] = {"bfs_levels_equal_oracle_8_sources": bfs_ok, "sssp_equal_oracle_4_sources": sssp_ok}
    # one Sampling-based Reordering round on a copy of the graph (C3-style reorder on/off)
    with sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), symmetric=True,
                       stream=stream.cuda_stream) as H:
        H.reorder(1)                 # warm-up round (first call builds the resident log, grows the pool)
        ob0 = H.objective(8)
        _, _, b0 = H.bfs(int(srcs[1]), out=level, push_only=True)
        st = H.reorder(1)
        ob1 = H.objective(8)
        _, _, b1 = H.bfs(int(srcs[1]), out=level, push_only=True)
        ex["reorder"] = {"round_ms": st["ms"], "note": "second round on the graph (first round = warm-up)", "swaps": st["vertices_discovered"], "movers": st["vertices_expanded"],
                         "objective_before": ob0, "objective_after": ob1,
                         "bfs_push_ms_before": b0["kernel_ms"], "bfs_push_ms_after": b1["kernel_ms"]}
        # online sampling (NEXT #3): 4 BFS queries recording their rows, threshold |E| -> a round
        # after every query that crosses it; wall time of each sage_bfs call incl. recording + round
        H.online_reorder(True, 8, 0)
        walls = []
        for i in range(4):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            _, _, bs = H.bfs(int(srcs[2 + i]), out=level, push_only=True)
            torch.cuda.synchronize()
            walls.append((time.perf_counter() - t0) * 1e3)
        info = H.online_info()
        H.online_reorder(False)
        ex["online_reorder"] = {"bfs_call_wall_ms": walls, "rounds": info["rounds"], "swaps": info["swaps"],
                                "threshold": "|E|", "note": "each call = BFS + row recording (+ one round "
                                "when the recorded row lengths reach |E|)"}
    return ex


if __name__ == "__main__":
    main()
