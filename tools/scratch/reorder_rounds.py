"""Per-round reorder time on C3 over 6 back-to-back rounds (no queries between)."""
import os, sys, time
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_sigmod_00020t21_b200 as sage
import sagegen as sg
g = sg.config("C3")
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda())
del g
for r in range(6):
    t0 = time.perf_counter()
    st = G.reorder(1)
    print(f"round {r}: event {st['ms']:.0f} ms, kernel {st.get('kernel_ms', 0):.0f} ms, wall {1e3 * (time.perf_counter() - t0):.0f} ms, swaps {st.get('vertices_discovered')}", flush=True)
