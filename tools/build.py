"""Native build for the three shared libraries of this repo.

* ``paper_conf_sigmod_00020t21_b200/libsage.so``  — the product: CUDA kernels for sm_100a +
  the C ABI declared in ``include/sage.h`` (nvcc, ``-gencode arch=compute_100a,code=sm_100a``).
* ``oracle/liboracle.so`` — the serial CPU oracle (plain C, gcc).  Test infrastructure.
* ``sagegen/libsagegen.so`` — seeded input generators (C++/OpenMP).  Test infrastructure.
* ``sagegen/libsagegen_dev.so`` — the same RMAT/Kronecker generator per rank on the device
  (CUDA; multi-GPU bench inputs such as C5).  Test / bench infrastructure.

The three share no source file and no header.  Builds are incremental (mtime based) and
in-tree so the ``.so`` files travel to the GPU box with the repo snapshot.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sigmod_00020t21_b200")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_paths():
    """NCCL headers/libs: prefer the copy torch loads (same soname, one NCCL per process)."""
    try:
        import nvidia.nccl  # type: ignore

        base = list(nvidia.nccl.__path__)[0]
        inc, lib = os.path.join(base, "include"), os.path.join(base, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc, lib
    except Exception:
        pass
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


def _stale(target, sources):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd):
    r = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
    if r.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + r.stdout)
        raise RuntimeError("build failed: " + cmd[0])
    return r.stdout


def build_sagegen(force=False):
    src = os.path.join(ROOT, "sagegen", "sagegen.cpp")
    out = os.path.join(ROOT, "sagegen", "libsagegen.so")
    if force or _stale(out, [src]):
        _run(["g++", "-O3", "-march=x86-64-v2", "-std=c++17", "-fopenmp", "-shared", "-fPIC", src, "-o", out])
    return out


def build_sagegen_dev(force=False):
    """Per-rank device generator of the RMAT / Kronecker inputs (bench + tests infrastructure)."""
    src = os.path.join(ROOT, "sagegen", "sagegen_dev.cu")
    out = os.path.join(ROOT, "sagegen", "libsagegen_dev.so")
    if force or _stale(out, [src]):
        _run([NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC", "-shared", src, "-o", out])
    return out


def build_oracle(force=False):
    src = os.path.join(ROOT, "oracle", "oracle.c")
    out = os.path.join(ROOT, "oracle", "liboracle.so")
    if force or _stale(out, [src]):
        # -O2, no -ffast-math: the oracle's fp64 arithmetic stays IEEE and in source order.
        _run(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", src, "-o", out, "-lm"])
    return out


def build_sage(force=False, verbose=False):
    csrc = os.path.join(PKG, "csrc")
    cus = sorted(glob.glob(os.path.join(csrc, "*.cu")))
    hdrs = (sorted(glob.glob(os.path.join(csrc, "*.cuh"))) + sorted(glob.glob(os.path.join(csrc, "*.h"))) +
            [os.path.join(ROOT, "include", "sage.h")])
    prof = os.environ.get("SAGE_PROF") == "1"
    out = os.path.join(PKG, "libsage_prof.so" if prof else "libsage.so")
    # compile-time variants (SAGE_DEF_NAME=VALUE -> -DNAME=VALUE, used by the A/B scripts): the
    # active set is stamped next to the library and its objects, and a different set is stale
    defs = sorted(f"-D{k[len('SAGE_DEF_'):]}={v}" for k, v in os.environ.items() if k.startswith("SAGE_DEF_"))
    if prof:
        defs.append("-DSAGE_PROF=1")
    stamp = out + ".defs"
    want = " ".join(defs) + "\n"
    have = open(stamp).read() if os.path.exists(stamp) else None
    if have != want:
        force = True
    if not (force or _stale(out, cus + hdrs)):
        return out
    nccl_inc, nccl_lib = _nccl_paths()
    objdir = os.path.join(PKG, "build_prof" if prof else "build")
    os.makedirs(objdir, exist_ok=True)
    common = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC",
              "-I", os.path.join(ROOT, "include"), "-I", csrc, "-I", nccl_inc,
              "--expt-relaxed-constexpr", "-Xptxas", "-v" if verbose else "-O3"] + defs
    objs = []
    for cu in cus:
        obj = os.path.join(objdir, os.path.basename(cu)[:-3] + ".o")
        if force or _stale(obj, [cu] + hdrs):
            log = _run(common + ["-c", cu, "-o", obj])
            if verbose:
                sys.stdout.write(log)
        objs.append(obj)
    if os.path.exists(stamp):
        os.remove(stamp)
    _run([NVCC, *ARCH, "-shared", "-o", out, *objs, "-L", nccl_lib, "-l:libnccl.so.2",
          "-Xlinker", "-rpath=" + nccl_lib])
    with open(stamp, "w") as f:
        f.write(want)
    return out


def build_all(force=False, verbose=False):
    return [build_sagegen(force), build_sagegen_dev(force), build_oracle(force), build_sage(force, verbose)]


if __name__ == "__main__":
    for p in build_all(force="--force" in sys.argv, verbose="-v" in sys.argv):
        print(p)
