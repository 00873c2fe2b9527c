"""Full-size BASELINE configs on one B200 with the CPU oracle beside them (not part of bench.py,
which times C2): C3 (twitter-like, 41.6M vertices, ~1.4B arcs) push BFS, and C4 (UK-2007-like,
105M vertices, ~3.7B arcs, >500 levels) push BFS + 20-iteration PageRank.  BFS levels are
compared element by element with oracle.bfs on 2 sources; PageRank with oracle.pagerank
(max relative error); GPU times are CUDA-event times of the sage_* calls (graph resident).
Usage: python tools/full_configs.py C3 C4 > gpurun_out/full_configs.json"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402


def run(cfg):
    t0 = time.time()
    g = sg.config(cfg)
    res = {"config": cfg, "graph": g.name, "n": g.n, "arcs": g.m, "gen_s": round(time.time() - t0, 1),
           "max_out_degree": int(np.diff(g.off).max())}
    srcs = [int(s) for s in sg.sources(g, 4, seed=2)]
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    off_d, col_d = torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda()
    G = sage.load_csr(off_d, col_d, borrow=True, stream=stream.cuda_stream)
    lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
    G.bfs(srcs[0], out=lv, push_only=True)           # warm-up (allocates the query state)
    bfs = []
    for i, s in enumerate(srcs):
        _, _, st = G.bfs(s, out=lv, push_only=True)
        rec = {"source": s, "kernel_ms": st["kernel_ms"], "ms": st["ms"], "levels": st["levels"],
               "edges": st["edges_traversed"], "gteps": st["edges_traversed"] / (st["ms"] * 1e-3) / 1e9,
               "model_GBps": (st["model_bytes"]) / (st["kernel_ms"] * 1e-3) / 1e9}
        if i < 2:
            got = lv.cpu().numpy()
            t1 = time.time()
            ref = oracle.bfs(g.off, g.col, s)
            rec["oracle_s"] = round(time.time() - t1, 2)
            rec["oracle_gteps"] = st["edges_traversed"] / rec["oracle_s"] / 1e9
            rec["levels_equal_oracle"] = bool(np.array_equal(got, ref))
        bfs.append(rec)
    res["bfs_push"] = bfs
    if cfg == "C4":
        x = torch.empty(g.n, dtype=torch.float64, device="cuda")
        pr = []
        for r in range(3):
            _, st = G.pagerank(0.85, 20, out=x)
            pr.append(st["ms"])
        res["pagerank_20_ms"] = pr
        res["pagerank_form"] = ("push (Alg. 1 l.26-29), windowed: near targets in a shared-memory fp64 window, "
                                "heavy far targets in a shared hot table, the rest fp64 reductions in global memory"
                                if G.pagerank_windowed else
                                "push (Alg. 1 l.26-29), fp64 reductions over the resident all-V log")
        xl = torch.empty_like(x)
        _, stl = G.pagerank(0.85, 20, out=xl, stealing=False)
        res["pagerank_log_form_ms_per_iteration"] = stl["ms"] / 20
        res["pagerank_log_form_max_rel_diff"] = float(((xl - x).abs() / x).max())
        res["pagerank_ms_per_iteration"] = min(pr) / 20
        res["pagerank_GBps_model"] = 20 * (40.0 * g.n + 12.0 * g.m) / (min(pr) * 1e-3) / 1e9
        t1 = time.time()
        xr = oracle.pagerank(g.off, g.col, 0.85, 20)
        res["pagerank_oracle_s"] = round(time.time() - t1, 1)
        xg = x.cpu().numpy()
        res["pagerank_max_rel_err"] = float(np.max(np.abs(xg - xr) / xr))
        res["pagerank_sum"] = float(xg.sum())
    G.free()
    return res


if __name__ == "__main__":
    out = {"host_cpus": os.cpu_count(), "gpu": torch.cuda.get_device_name(0)}
    try:
        out["host_mem_gb"] = round(os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES") / 2**30, 1)
    except (ValueError, OSError):
        pass
    for cfg in sys.argv[1:] or ["C3", "C4"]:
        out[cfg] = run(cfg)
        print(json.dumps(out), flush=True)
