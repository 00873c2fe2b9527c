"""C1 (RMAT-16) per-call latency vs grid size (sage_options.ctas_per_sm) and hub filter; L2 flushed
between calls like bench.py.  Usage (GPU): python tools/c1_sweep.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

g = sg.config("C1")
s = torch.cuda.Stream()
torch.cuda.set_stream(s)
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
src = sg.sources(g, 16, seed=2)
lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
for cps in (0, 1, 2):
    G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda(), symmetric=True,
                      stream=s.cuda_stream, ctas_per_sm=cps)
    for po in (True, False):
        G.bfs(int(src[0]), out=lv, push_only=po)
        ev, ks = [], []
        for i, x in enumerate(src):
            flush.fill_(float(i))
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s)
            _, _, st = G.bfs(int(x), out=lv, push_only=po)
            e1.record(s)
            e1.synchronize()
            ev.append(e0.elapsed_time(e1) * 1e3)
            ks.append(st["kernel_ms"] * 1e3)
        rec = G.level_records()
        print(f"ctas_per_sm={cps} {'push' if po else 'do  '}: call {np.median(ev):7.1f} us  kernel {np.median(ks):7.1f} us"
              f"  levels {st['levels']}  level us {np.round(np.diff(np.concatenate([[0], rec[:, 6]])) / 1e3, 1)}")
    G.free()
