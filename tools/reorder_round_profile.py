"""One Sampling-based Reordering round on C3 (twitter-like) inside a cudaProfilerStart/Stop range, for
`ncu --profile-from-start off --metrics gpu__time_duration.sum` launch lists (the round's kernel split).
Usage: python tools/reorder_round_profile.py [n_vertices]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sigmod_00020t21_b200 as sage  # noqa: E402
import sagegen as sg  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 0
g = sg.config("C3") if not n else sg.twitter_like(n=n, tuples=n * 38, seed=1)
G = sage.load_csr(torch.from_numpy(g.off).cuda(), torch.from_numpy(g.col).cuda())
del g
print("warm-up round", G.reorder(1)["ms"], "ms", flush=True)
torch.cuda.synchronize()
torch.cuda.profiler.start()
st = G.reorder(1)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("profiled round", st["ms"], "ms")
