import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import oracle, sagegen as sg
import paper_conf_sigmod_00020t21_b200 as sage
g = sg.rmat(16, 16, seed=9, symmetric=True)
w = sg.weights(g, 3)
srcs = [int(x) for x in sg.sources(g, 3, seed=4)]
with sage.load_csr(g.off, g.col, w, symmetric=True) as G:
    for rnd in range(2):
        for s in srcs:
            ref = oracle.bfs(g.off, g.col, s)
            for po in (True, False):
                for direct in (True, False):
                    if direct:
                        lv = torch.full((g.n,), 12345, dtype=torch.int32, device="cuda")
                        par = torch.full((g.n,), 777, dtype=torch.int32, device="cuda")
                        G.bfs(s, out=lv, parent_out=par, push_only=po)
                        lvn, parn = lv.cpu().numpy(), par.cpu().numpy()
                    else:
                        lvn, parn, _ = G.bfs(s, parents=True, push_only=po)
                    print(rnd, s, "push" if po else "do", "direct" if direct else "host", "lv ok", np.array_equal(lvn, ref), "par[src]", parn[s], "unreached par vals", np.unique(parn[ref < 0])[:5])
            G.sssp(s)
        if rnd == 0:
            G.reorder(rounds=1)
