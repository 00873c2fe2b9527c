"""Push-BFS kernel time on a full-size config (no oracle): python tools/cfg_bfs.py C4 [reps]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 4
g = sg.config(cfg)
srcs = [int(s) for s in sg.sources(g, reps, seed=2)]
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), symmetric=g.symmetric)
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
G.bfs(srcs[0], out=lv, push_only=True)
ks = [G.bfs(s, out=lv, push_only=True)[2]["kernel_ms"] for s in srcs]
print(json.dumps({"config": cfg, "kernel_ms": [round(k, 3) for k in ks], "mean": float(np.mean(ks))}))
