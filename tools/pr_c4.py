"""C4 (UK-2007-like, 105M vertices, ~3.7e9 arcs) push PageRank timing: ms per iteration over
`iters` iterations after a 2-iteration warm-up (graph resident; the log built in the warm-up).
Usage: python tools/pr_c4.py [iters] [n]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

iters = int(sys.argv[1]) if len(sys.argv) > 1 else 5
n = int(sys.argv[2]) if len(sys.argv) > 2 else 105_000_000
t0 = time.time()
g = sg.uk_like(n=n, seed=1) if n != 105_000_000 else sg.config("C4")
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), stream=stream.cuda_stream)
x = torch.empty(g.n, dtype=torch.float64, device="cuda")
res = {"graph": g.name, "n": g.n, "arcs": g.m, "iters": iters, "gen_s": round(time.time() - t0, 1)}
for form, stealing in (("windowed", True),) + ((("log", False),) if not os.environ.get("PR_WIN_ONLY") else ()):
    G.pagerank(0.85, 2, out=x, stealing=stealing)
    _, st = G.pagerank(0.85, iters, out=x, stealing=stealing)
    res[form] = {"ms_per_iteration": st["kernel_ms"] / iters,
                 "model_GBps": st["model_bytes"] / (st["kernel_ms"] * 1e-3) / 1e9}
    if stealing:
        res[form]["selected"] = G.pagerank_windowed
        xw = x.cpu()
    else:
        res["max_rel_diff_windowed_vs_log"] = float(((xw - x.cpu()).abs() / x.cpu()).max())
print(json.dumps(res))
