"""Fig. 10-style ablation on B200: push-only BFS on C2 (RMAT-24) with
   1. no Tiled Partitioning: ladder B = M = 4096 — rows below 4096 arcs are consumed by the warp
      scan-based gather only (Merrill-style load balancing, the paper's [30]),
   2. Tiled Partitioning without Resident Tile Stealing (static round-robin tile assignment),
   3. TP + RTS (the default),
   4. TP + RTS after Sampling-based Reordering (1 and 4 rounds).
Prints one JSON object (mean kernel ms over the same sources, GTEPS)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
g = sg.rmat(scale, 16, 1, True)
srcs = [int(s) for s in sg.sources(g, 4, seed=2)]
off = torch.from_numpy(g.off).cuda()
col = torch.from_numpy(g.col).cuda()
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
out = {"graph": f"rmat{scale} sym", "arcs": g.m}


def run(G, **kw):
    G.bfs(srcs[0], out=lv, push_only=True, **kw)
    ms, edges = [], []
    for s in srcs:
        _, _, st = G.bfs(s, out=lv, push_only=True, **kw)
        ms.append(st["kernel_ms"])
        edges.append(st["edges_traversed"])
    return {"kernel_ms": float(np.mean(ms)), "gteps": float(np.sum(edges) / (np.sum(ms) * 1e-3) / 1e9)}


with sage.load_csr(off, col, symmetric=True, tile_cta=4096, tile_min=4096, align=0) as G:
    out["1_no_TP_scan_gather_only"] = run(G)
with sage.load_csr(off, col, symmetric=True) as G:
    out["2_TP_no_RTS"] = run(G, stealing=False)
    out["3_TP_RTS"] = run(G)
    G.reorder(1)
    out["4_TP_RTS_SR1"] = run(G)
    G.reorder(3)
    out["4_TP_RTS_SR4"] = run(G)
print(json.dumps(out))
