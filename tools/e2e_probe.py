"""e2e probe: time each part of the end-to-end BFS call chain (pinned host CSR -> load -> BFS -> D2H)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sigmod_00020t21_b200 as sage, sagegen as sg
g = sg.config("C2")
off_h = torch.from_numpy(g.off).pin_memory(); col_h = torch.from_numpy(g.col).pin_memory()
lv_h = torch.empty(g.n, dtype=torch.int32).pin_memory()
src = sg.sources(g, 4, seed=2)
for i in range(4):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    H = sage.load_csr(off_h, col_h, symmetric=True)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    _, _, st = H.bfs(int(src[i]), out=lv_h, push_only=True)
    torch.cuda.synchronize(); t2 = time.perf_counter()
    H.free(); torch.cuda.synchronize(); t3 = time.perf_counter()
    print(f"load {1e3*(t1-t0):.1f} ms  bfs call {1e3*(t2-t1):.1f} ms (kernel {st['kernel_ms']:.2f}, ms {st['ms']:.2f})  free {1e3*(t3-t2):.1f} ms")
