import sys, time, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_sigmod_00020t21_b200 as sage, sagegen as sg
g = sg.config("C1")
s = torch.cuda.current_stream()
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), symmetric=True, stream=s.cuda_stream)
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
src = sg.sources(g, 16, seed=2)
for po in (True, False):
    G.bfs(int(src[0]), out=lv, push_only=po)
    ks, ms, walls = [], [], []
    for x in src:
        torch.cuda.synchronize(); t0 = time.perf_counter()
        _, _, st = G.bfs(int(x), out=lv, push_only=po)
        walls.append((time.perf_counter() - t0) * 1e6)
        ks.append(st["kernel_ms"] * 1e3); ms.append(st["ms"] * 1e3)
    print("push_only" if po else "do", "kernel us", np.median(ks), "call(event) us", np.median(ms), "wall us", np.median(walls), "levels", st["levels"])
    rec = G.level_records()
    print("  level t_ns deltas us:", np.diff(np.concatenate([[0], rec[:, 6]])) / 1e3)
