import os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_sigmod_00020t21_b200 as sage, sagegen as sg
stream = torch.cuda.Stream(); torch.cuda.set_stream(stream)
g = sg.config("C2")
srcs = sg.sources(g, 4, seed=2)
level = torch.empty(g.n, dtype=torch.int32, device="cuda")
def probe(tag):
    with sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), symmetric=True,
                       stream=stream.cuda_stream) as H:
        t0 = time.perf_counter(); st0 = H.reorder(1); w0 = time.perf_counter() - t0
        ob0 = H.objective(8)
        H.bfs(int(srcs[1]), out=level, push_only=True)
        t0 = time.perf_counter(); st = H.reorder(1); w1 = time.perf_counter() - t0
        t0 = time.perf_counter(); st2 = H.reorder(1); w2 = time.perf_counter() - t0
        print(tag, "round ms", st0["ms"], st["ms"], st2["ms"], "wall s", w0, w1, w2, flush=True)
probe("alone")
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), torch.from_numpy(g.w).cuda(),
                  symmetric=True, borrow=True, stream=stream.cuda_stream)
for i in range(3):
    G.bfs(int(srcs[i]), out=level, push_only=True)
probe("with C2 loaded")
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
probe("with flush buf")
