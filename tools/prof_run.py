"""Profiling driver: load a graph once and run a few queries (used under ncu; not a bench)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("--scale", type=int, default=24)
p.add_argument("--graph", default="rmat", choices=["rmat", "uk", "twitter"])
p.add_argument("--n", type=int, default=0, help="vertices for uk / twitter shapes")
p.add_argument("--op", default="bfs_push", choices=["bfs_push", "bfs_do", "sssp", "pr", "pr_push", "reorder", "bc"])
p.add_argument("--reps", type=int, default=3)
p.add_argument("--tile-cta", type=int, default=256)
p.add_argument("--align", type=int, default=4)
a = p.parse_args()
if a.graph == "rmat":
    g = sg.rmat(a.scale, 16, 1, True)
elif a.graph == "uk":
    g = sg.uk_like(n=a.n or 10_000_000, seed=1, n_tendrils=200)
else:
    g = sg.twitter_like(n=a.n or 4_000_000, tuples=(a.n or 4_000_000) * 36, seed=1)
w = sg.weights(g, 1)
s = stream = torch.cuda.Stream()   # the library's work and the events on one stream
torch.cuda.set_stream(stream)
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), torch.from_numpy(w).cuda(),
                  symmetric=g.symmetric, borrow=True, stream=stream.cuda_stream, tile_cta=a.tile_cta, align=a.align)
src = sg.sources(g, a.reps, seed=2)
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
for i in range(a.reps):
    if a.op == "bfs_push":
        _, _, st = G.bfs(int(src[i]), out=lv, push_only=True)
    elif a.op == "bfs_do":
        _, _, st = G.bfs(int(src[i]), out=lv)
    elif a.op == "sssp":
        _, st = G.sssp(int(src[i]), out=lv.view(torch.uint32))
    elif a.op == "reorder":
        st = G.reorder(1)
    elif a.op == "bc":
        _, st = G.bc([int(src[i])])
    else:
        x = torch.empty(g.n, dtype=torch.float64, device="cuda")
        _, st = G.pagerank(0.85, 5, out=x, push_only=(a.op == "pr_push"))
    print(a.op, i, {k: st[k] for k in ("levels", "kernel_ms", "ms", "edges_traversed", "model_bytes")}, flush=True)
    if a.op not in ("pr", "pr_push", "reorder", "bc") and os.environ.get("LEVELS", "1") == "0":
        rec = G.level_records()
        dt = np.diff(np.concatenate([[0], rec[:, 6]])) / 1e3
        small = dt[rec[:, 2] < 10000]
        print("   levels=%d  median small-level us=%.1f  total small-level ms=%.2f" % (len(rec), np.median(small) if len(small) else 0, small.sum() / 1e3))
    if a.op not in ("pr", "pr_push", "reorder", "bc") and os.environ.get("LEVELS", "1") == "1":
        prev = 0
        for r in G.level_records():
            print("   L dir=%d |F|=%9d arcsF=%11d insp=%11d disc=%9d  %8.1f us (work done at +%8.1f, phase1 +%8.1f)" % (
                r[0], r[1], r[2], r[3], r[5], (r[6] - prev) / 1e3, (r[7] - prev) / 1e3, (r[8] - prev) / 1e3 if r[8] else 0))
            prev = r[6]
    if os.environ.get("SAGE_PROF") == "1":
        import ctypes
        buf = (ctypes.c_ulonglong * 16)()
        sage.lib().sage_prof_read(buf, 1)
        names = ["flush_cyc", "flushes", "visit_contig_cyc", "visit_strided_cyc", "strided_steps", "ticket_cyc",
                 "tickets", "_", "L1_sum_ns", "L1_max_ns", "L1_warps_gt20us", "L1_warps", "L1_start_max", "L1_start_min"]
        d = {nm: buf[k] for k, nm in enumerate(names)}
        print("   prof:", d, {"cyc/flush": d["flush_cyc"] / max(1, d["flushes"]),
                               "cyc/strided_step": d["visit_strided_cyc"] / max(1, d["strided_steps"]),
                               "cyc/ticket": d["ticket_cyc"] / max(1, d["tickets"])})
