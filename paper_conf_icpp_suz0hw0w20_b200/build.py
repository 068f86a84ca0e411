"""Build libsptrsv.so in-tree for sm_100a (nvcc; no JIT cache, no torch extension).

    python paper_conf_icpp_suz0hw0w20_b200/build.py          # or __graft_entry__.build()
(run it by path: importing the package loads the library this script builds)
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libsptrsv.so")
SOURCES = [os.path.join(CSRC, f) for f in ("sptrsv.cu",)]
DEPS = SOURCES + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + [os.path.join(ROOT, "include", "sptrsv.h")]
# ptxas register / spill report of the last build (untracked: build() must not dirty the tree)
PTXAS_INFO = os.path.join(ROOT, "build", "ptxas_info.txt")

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


def build(force: bool = False, verbose: bool = False, defines=()) -> str:
    if not force and not stale():
        return LIB
    tmp = LIB + ".tmp.%d" % os.getpid()
    cmd = [nvcc(), *NVCC_FLAGS, *("-D" + d for d in defines), "-I", os.path.join(ROOT, "include"), "-I", CSRC,
           "-o", tmp, *SOURCES]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed building libsptrsv.so")
    if verbose:
        sys.stderr.write(res.stderr)
    os.makedirs(os.path.dirname(PTXAS_INFO), exist_ok=True)
    with open(PTXAS_INFO, "w") as f:
        f.write(res.stderr)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True,
          defines=[a[2:] for a in sys.argv[1:] if a.startswith("-D")])
    print(LIB)
