"""Build libclover.so (the C-ABI library, include/clover.h) in-tree with nvcc
for sm_100a.  Called by __graft_entry__.build() and by the binding when the
library is missing or stale.

Flags: -fmad=false keeps every fp64 multiply and add separately rounded
(reading A8: bitwise parity with any IEEE implementation of the
same reading); -lineinfo for ncu source mapping.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libclover.so")
ARCH = "-gencode=arch=compute_100a,code=sm_100a"


def nccl_dir() -> str | None:
    for p in sys.path:
        d = os.path.join(p, "nvidia", "nccl")
        if os.path.exists(os.path.join(d, "include", "nccl.h")) and \
                os.path.exists(os.path.join(d, "lib", "libnccl.so.2")):
            return d
    return None


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.sep not in c or os.path.exists(c)):
            return c
    return "nvcc"


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                  [os.path.join(ROOT, "include", "clover.h")])


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def build(force: bool = False, verbose: bool = False, out: str | None = None,
          defines: tuple = ()) -> str:
    """Build libclover.so (or a variant at `out` with extra -D defines, for
    A/B experiments: scripts/ab_variants.py)."""
    target = out or LIB
    if out is None and not force and not stale():
        return LIB
    cmd = [nvcc(), "-O3", "-std=c++17", ARCH, "-lineinfo", "-fmad=false",
           "-Xcompiler", "-fPIC", "-shared", "-I", os.path.join(ROOT, "include"),
           "-o", target + ".tmp", os.path.join(CSRC, "clover_engine.cu")]
    cmd += ["-D" + d for d in defines]
    nd = nccl_dir()
    if nd:
        cmd += ["-DCLOVER_WITH_NCCL", "-I", os.path.join(nd, "include"),
                "-L", os.path.join(nd, "lib"), "-l:libnccl.so.2",
                "-Xlinker", "-rpath=" + os.path.join(nd, "lib")]
    if verbose:
        cmd += ["-Xptxas", "-v"]
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
