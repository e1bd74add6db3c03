"""In-tree build of libsssp.so for sm_100a (nvcc; no JIT cache, no torch extension).

The .so files land next to this file so they travel with the repo snapshot to
the GPU box and are the ones the tests/bench load:

  libsssp.so       the product library
  libsssp_fuzz.so  the same sources with -DSSSP_FUZZ: hash-driven __nanosleep
                   delays at the worklist's reserve / publish / claim / complete /
                   head-CAS points (schedule fuzzing for the parity tests only)
"""
from __future__ import annotations

import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libsssp.so")
VARIANTS = {"": [], "fuzz": ["-DSSSP_FUZZ"]}
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-lineinfo", "-O3", "-std=c++17",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-O3",
    "-shared",
    f"-I{os.path.join(ROOT, 'include')}",
]


def variant_path(variant: str = "") -> str:
    return LIB if not variant else os.path.join(HERE, f"libsssp_{variant}.so")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def deps():
    return sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h"))) + [
        os.path.join(ROOT, "include", "sssp.h"), __file__]


def stale(variant: str = "") -> bool:
    p = variant_path(variant)
    if not os.path.exists(p):
        return True
    t = os.path.getmtime(p)
    return any(os.path.getmtime(d) > t for d in deps())


def build(force: bool = False, verbose: bool = False, variants=None) -> str:
    """Compile every variant that is missing or stale (in parallel)."""
    procs = []
    for v in (VARIANTS if variants is None else variants):
        if not force and not stale(v):
            continue
        out = variant_path(v)
        tmp = out + f".tmp{os.getpid()}"
        cmd = [NVCC, *NVCC_FLAGS, *VARIANTS[v], "-o", tmp, *sources()]
        if verbose and not v:
            cmd.insert(1, "-Xptxas=-v")
        procs.append((subprocess.Popen(cmd), tmp, out))
    for p, tmp, out in procs:
        if p.wait() != 0:
            raise subprocess.CalledProcessError(p.returncode, "nvcc")
        os.replace(tmp, out)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
