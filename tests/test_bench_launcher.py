"""Host logic of bench.py's multi-GPU mode (CPU; no GPU needed).

* `--gpus N` outside torchrun re-launches itself as N ranks through torch.distributed.run on
  127.0.0.1 (and does nothing under torchrun or for N = 1);
* the weak-scaling workload: Kronecker scale 24 + log2(N) (C2 at N = 1), 27 + log2(N) for C5;
* the seeded sources of a 1D-partitioned graph (allgathered non-empty flags, world 2 on gloo)
  equal sagegen.sources on the whole graph.
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import sagegen as sg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


class _A:
    def __init__(self, gpus):
        self.gpus = gpus


def test_spawn_command(monkeypatch):
    calls = []
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(bench.subprocess, "call", lambda cmd: calls.append(cmd) or 0)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "4", "--steps", "3"])
    assert bench._spawn_if_needed(_A(4)) == 0
    cmd = calls[0]
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "--master-addr=127.0.0.1" in cmd and "--nnodes=1" in cmd
    assert cmd[-4:] == ["--gpus", "4", "--steps", "3"] and cmd[-5].endswith("bench.py")
    assert bench._spawn_if_needed(_A(1)) is None
    monkeypatch.setenv("WORLD_SIZE", "4")
    assert bench._spawn_if_needed(_A(4)) is None


def test_weak_scaling_workload():
    assert [bench.multi_workload("C2", n) for n in (1, 2, 4, 8)] == [24, 25, 26, 27]
    assert [bench.multi_workload("C5", n) for n in (1, 2, 4, 8)] == [27, 28, 29, 30]
    with pytest.raises(ValueError):
        bench.multi_workload("C2", 3)


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = sg.rmat(10, 4, seed=5, symmetric=False)        # directed: some rows are empty
    n = g.n
    vb, ve = n * rank // world, n * (rank + 1) // world
    off = torch.from_numpy(g.off[vb:ve + 1] - g.off[vb])
    s = bench._nonempty_sources(torch, off, n, world, 12)
    q.put((rank, s.tolist()))
    dist.destroy_process_group()


def test_partitioned_sources_equal_sagegen():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(60)
    g = sg.rmat(10, 4, seed=5, symmetric=False)
    ref = sg.sources(g, 12, seed=2).tolist()
    assert res[0] == ref and res[1] == ref
