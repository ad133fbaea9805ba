"""nvcc build of libugache.so (in-tree, sm_100a only)."""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
OUT = os.path.join(PKG, "libugache.so")
SOURCES = [os.path.join(CSRC, "ugache.cu"), os.path.join(CSRC, "solver.cc")]
DEPS = SOURCES + [os.path.join(CSRC, "kernels.cuh"), os.path.join(CSRC, "ugache_internal.h"),
                  os.path.join(INCLUDE, "ugache.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def command(out: str = OUT):
    return [NVCC, "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
            "-lineinfo", "-Xptxas", "-v", "-Xcompiler", "-fPIC,-fopenmp,-O3,-Wall",
            "-shared", f"-I{INCLUDE}", "-o", out] + SOURCES + ["-lgomp"]


def build(force: bool = False, verbose: bool = False) -> str:
    stale = (not os.path.exists(OUT) or
             any(os.path.getmtime(d) > os.path.getmtime(OUT) for d in DEPS))
    if force or stale:
        log = os.path.join(PKG, "build.log")
        with open(log, "w") as f:
            r = subprocess.run(command(), stdout=f, stderr=subprocess.STDOUT)
        if r.returncode != 0:
            sys.stderr.write(open(log).read())
            raise RuntimeError(f"nvcc failed, see {log}")
        if verbose:
            sys.stdout.write(open(log).read())
    return OUT


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
