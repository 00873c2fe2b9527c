"""C3 (BASELINE configs[2]): twitter-like graph at full size (41.6M vertices, ~1.46B arcs),
push-only BFS before and after Sampling-based Reordering rounds {1, 5, 20, 99} (the paper's
SAGE_1 ... SAGE_100), with the per-round reorder time and the tile-sector objective.
BFS answers (original ids) must not change across rounds (checked)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

rounds_max = int(sys.argv[1]) if len(sys.argv) > 1 else 99
t0 = time.time()
g = sg.config("C3")
out = {"graph": f"twitter_like n={g.n} arcs={g.m}", "gen_s": time.time() - t0,
       "max_out_degree": int(np.diff(g.off).max())}
srcs = [int(s) for s in sg.sources(g, 4, seed=2)]
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda())
del g


def bfs_all():
    ms, te, lvls = [], [], []
    for s in srcs:
        _, _, st = G.bfs(s, out=lv, push_only=True)
        ms.append(st["kernel_ms"])
        te.append(st["edges_traversed"])
        lvls.append(lv.cpu().numpy().copy())
    return {"kernel_ms": float(np.mean(ms)), "gteps": float(np.sum(te) / (np.sum(ms) * 1e-3) / 1e9)}, lvls


G.bfs(srcs[0], out=lv, push_only=True)
res, ref = bfs_all()
res["objective"] = G.objective(8)
out["rounds_0"] = res
done, round_ms = 0, []
for target in [1, 5, 20, 99]:
    if target > rounds_max:
        break
    while done < target:
        st = G.reorder(1)
        round_ms.append(st["ms"])
        done += 1
        if st["vertices_discovered"] == 0:
            break
    res, lvls = bfs_all()
    res["objective"] = G.objective(8)
    res["answers_unchanged"] = all(np.array_equal(a, b) for a, b in zip(lvls, ref))
    res["rounds_done"] = done
    out[f"rounds_{target}"] = res
out["reorder_round_ms"] = {"first": round_ms[0], "median_after_first": float(np.median(round_ms[1:])) if len(round_ms) > 1 else None}
print(json.dumps(out))
