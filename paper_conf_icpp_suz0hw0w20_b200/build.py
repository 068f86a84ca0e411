"""Build libsptrsv.so in-tree for sm_100a (nvcc; no JIT cache, no torch extension).

    python paper_conf_icpp_suz0hw0w20_b200/build.py          # or __graft_entry__.build()
(run it by path: importing the package loads the library this script builds)
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libsptrsv.so")
SOURCES = [os.path.join(CSRC, f) for f in ("sptrsv.cu",)]
DEPS = SOURCES + [os.path.join(CSRC, f) for f in ("solve.cuh", "solve_pipe.cuh", "solve_k.cuh", "solve_dyn.cuh", "solve_lean.cuh", "solve_tri.cuh", "solve_multi.cuh", "solve_paper.cuh", "setup.cuh", "ptx.cuh", "diag.cuh")] + [
    os.path.join(ROOT, "include", "sptrsv.h")]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared",
    "-Xptxas", "-v",
    "--expt-relaxed-constexpr",
]


def nvcc() -> str:
    cand = os.path.join(os.environ.get("CUDA_HOME", "/usr/local/cuda"), "bin", "nvcc")
    return cand if os.path.exists(cand) else "nvcc"


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in DEPS)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    tmp = LIB + ".tmp.%d" % os.getpid()
    cmd = [nvcc(), *NVCC_FLAGS, "-I", os.path.join(ROOT, "include"), "-I", CSRC, "-o", tmp, *SOURCES]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed building libsptrsv.so")
    if verbose:
        sys.stderr.write(res.stderr)
    with open(os.path.join(CSRC, "ptxas_info.txt"), "w") as f:
        f.write(res.stderr)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
