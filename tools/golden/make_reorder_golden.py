"""Write tests/golden/reorder_<case>.json: the ORACLE's Sampling-based Reordering result on inputs
too large to recompute inside the GPU test run (RMAT-20, a 1M-vertex twitter-like graph).

Calls only oracle/ (plus the seeded input generator sagegen/, which holds no SAGE arithmetic).
Stored per case: the generator parameters, the ladder / sector width / rounds, the number of
relabelled vertices, SHA-256 digests of the permutation (int32 sigma[v], original id -> label) and
of the relabelled off / col / weights arrays, and the per-round info.  tests/test_gpu_reorder.py regenerates the graph, runs the GPU
reorder and compares.

    python tools/golden/make_reorder_golden.py [case ...]
"""
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import sagegen as sg  # noqa: E402

CASES = {
    "rmat20": dict(gen="rmat", scale=20, ef=16, seed=7, symmetric=True, rounds=1, B=256, M=8, A=4, S=8,
                   weights_seed=2),
    "twitter1m": dict(gen="twitter_like", n=1_000_000, tuples=36_000_000, seed=1, rounds=1, B=256, M=8, A=4,
                      S=8, weights_seed=None),
}


def graph(c):
    if c["gen"] == "rmat":
        g = sg.rmat(c["scale"], c["ef"], c["seed"], c["symmetric"])
    else:
        g = sg.twitter_like(n=c["n"], tuples=c["tuples"], seed=c["seed"])
    w = sg.weights(g, c["weights_seed"]) if c.get("weights_seed") else None
    return g, w


def digest(a):
    return hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()


def main(names):
    for name in names:
        c = CASES[name]
        g, w = graph(c)
        t0 = time.time()
        off2, col2, w2, sigma, info = oracle.reorder(g.off, g.col, w, rounds=c["rounds"], B=c["B"], M=c["M"],
                                                     A=c["A"], S=c["S"])
        dt = time.time() - t0
        moved = np.nonzero(sigma != np.arange(g.n))[0]
        out = {"citation": "oracle.reorder (oracle/oracle.c, SURVEY §8(c) c5: stages 1-3 P:418-442, swap "
                           "matching R23, sorted relabel R24) on a seeded sagegen input; written by "
                           "tools/golden/make_reorder_golden.py, which calls only oracle/",
               "case": c, "n": int(g.n), "m": int(g.m), "oracle_seconds": round(dt, 1),
               "n_moved": int(len(moved)), "sha256_sigma": digest(sigma.astype(np.int32)),
               "sha256_off": digest(off2), "sha256_col": digest(col2),
               "sha256_w": digest(w2) if w2 is not None else None,
               "info": [{k: int(v) for k, v in r.items()} for r in info]}
        p = os.path.join(ROOT, "tests", "golden", f"reorder_{name}.json")
        with open(p, "w") as f:
            json.dump(out, f, indent=1)
        print(name, g.n, g.m, f"{dt:.1f}s", len(moved), "moved", info, flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or list(CASES))
